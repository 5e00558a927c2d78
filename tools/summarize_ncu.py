"""Summarize a round's ncu captures (run here, no GPU): python tools/summarize_ncu.py r01"""
import csv, io, json, os, subprocess, sys
R = sys.argv[1] if len(sys.argv) > 1 else "r01"
OUT = "gpurun_out"
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__ops_path_tensor_op_utchmma_src_bf16_dst_fp32_sparsity_off.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__shared_mem_per_block_dynamic", "sm__cycles_elapsed.avg.per_second"]
summary = {"round": R, "kernels": {}}
for tag in ["memo_pair", "memo_ws", "brickify", "padded", "gen_cfg5", "gen_cfg4"]:
    rep = os.path.join(OUT, f"{R}_{tag}.ncu-rep")
    if not os.path.exists(rep):
        continue
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        name = r[hdr.index("Kernel Name")]
        d = {}
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                d[k] = {"value": r[i], "unit": units[i]}
        summary["kernels"].setdefault(name[:80], []).append(d)
    with open(f"profiles/{R}_{tag}_raw.csv", "w") as f:
        w = csv.writer(f)
        keep = [i for i, h in enumerate(hdr) if h in KEYS or h in ("Kernel Name", "ID")]
        for r in rows:
            w.writerow([r[i] for i in keep])
# launch list
lc = os.path.join(OUT, f"{R}_launches.csv")
if os.path.exists(lc):
    rows = list(csv.reader(open(lc)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    launches = [(r[ki], float(r[vi])) for r in rows[hi + 1:] if len(r) > vi]
    tot = {}
    for k, v in launches:
        key = k.split("(")[0]
        tot.setdefault(key, []).append(v)
    summary["launch_list"] = {k: {"count": len(v), "mean_ns": sum(v) / len(v)} for k, v in tot.items()}
    ours = {k: sum(v) for k, v in tot.items()
            if any(t in k for t in ("bdl::", "memo_ws", "memo_pair", "gen_kernel", "brickify", "pool_vec")) and "pack" not in k}
    s = sum(ours.values())
    summary["launch_share_of_step"] = {k: v / s for k, v in ours.items()}
    with open(f"profiles/{R}_launches.csv", "w") as f:
        f.write("kernel,duration_ns\n")
        for k, v in launches:
            f.write(f"\"{k[:90]}\",{v}\n")
# dram bytes per launch of the dominant kernel (for bench.py's roofline.traffic)
dram = None
for name, lst in summary["kernels"].items():
    if "memo_pair" in name or ("memo_ws" in name and dram is None):
        d = lst[0]
        rb = float(d["dram__bytes_read.sum"]["value"]) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[d["dram__bytes_read.sum"]["unit"]]
        wb = float(d["dram__bytes_write.sum"]["value"]) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[d["dram__bytes_write.sum"]["unit"]]
        dram = rb + wb
summary["dram_bytes_per_launch"] = {"tcgen05 band": dram}
json.dump(summary, open(f"profiles/{R}_summary.json", "w"), indent=1)
json.dump({"round": R, "dram_bytes_per_launch": {"tcgen05 band": dram}}, open("profiles/ncu_summary_latest.json", "w"), indent=1)
print(json.dumps(summary, indent=1)[:3000])
