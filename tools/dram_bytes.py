"""DRAM bytes of one forward pass: merged execution (this library) vs layer-by-layer torch/cuDNN (the Fig 9 analogue,
PAPER.md L1166-1377; SURVEY.md §8(d) "DRAM bytes vs layer-by-layer").

    # one forward inside an NVTX range, profiled by ncu (every kernel cold-cache, caches flushed between kernels):
    ncu --nvtx --nvtx-include "fwd/" --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
        --csv --log-file out.csv python tools/dram_bytes.py run --impl merged --config cfg4
    python tools/dram_bytes.py sum out.csv          # totals per kernel family
"""
import argparse
import csv
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(impl, cfg):
    import torch
    from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
    wl = workloads.make_workload(cfg)
    dev = torch.device("cuda")
    if impl == "merged":
        plan = engine.plan_from_workload(wl, device=dev)
        x = wl["x"].to(device=dev, dtype=plan.tdtype).contiguous()
        xb = plan.alloc_bricked(plan.in_layout)
        lo = plan.out_layout
        y = torch.empty((lo.N, lo.C, lo.D, lo.H, lo.W), dtype=plan.tdtype, device=dev)

        def fwd():
            plan.brickify(x, out=xb)
            plan.run_dense(xb, out=y)
    else:
        import torch.nn.functional as F
        nsp3 = wl["nsp"] == 3
        fmt = torch.channels_last_3d if nsp3 else torch.channels_last
        x = (wl["x"] if nsp3 else wl["x"][:, :, 0]).to(device=dev, dtype=torch.bfloat16).contiguous(memory_format=fmt)
        ws = [None if w is None else (w if nsp3 else w[:, :, 0]).to(device=dev, dtype=torch.bfloat16)
              .contiguous(memory_format=fmt) for w in wl["weights"]]
        bs = [None if b is None else b.to(device=dev, dtype=torch.bfloat16) for b in wl["biases"]]
        sl = slice(None) if nsp3 else slice(1, None)

        def fwd():
            outs = []
            for l, w, b in zip(wl["layers"], ws, bs):
                src = x if l["input"] == -1 else outs[l["input"]]
                if l["kind"] == "maxpool":
                    yy = (F.max_pool3d if nsp3 else F.max_pool2d)(src, l["k"][sl], l["stride"][sl], l["pad"][sl])
                else:
                    yy = (F.conv3d if nsp3 else F.conv2d)(src, w, b, stride=l["stride"][sl], padding=l["pad"][sl])
                if l["residual"] is not None:
                    yy = yy + (x if l["residual"] == -1 else outs[l["residual"]])
                if l["relu"]:
                    yy = torch.relu(yy)
                outs.append(yy)
            return outs[-1]
    with torch.no_grad():
        for _ in range(2):
            fwd()
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_push("fwd")
        fwd()
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_pop()


def summarize(path):
    rows = list(csv.reader(open(path)))
    i = next(k for k, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[i]
    tot = defaultdict(float)
    per = defaultdict(lambda: defaultdict(float))
    for r in rows[i + 1:]:
        if len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        name, metric, unit = d["Kernel Name"], d["Metric Name"], d["Metric Unit"]
        try:
            v = float(d["Metric Value"].replace(",", ""))
        except ValueError:
            continue
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
                 "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}.get(unit, 1)
        tot[metric] += v * scale
        per[name.split("(")[0].split("<")[0][:40]][metric] += v * scale
    n = len([r for r in rows[i + 1:] if len(r) == len(hdr)]) // 3
    return tot, per, n


def per_launch(path):
    """[(kernel name, DRAM bytes, duration s)] in launch order."""
    rows = list(csv.reader(open(path)))
    i = next(k for k, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[i]
    by = {}
    for r in rows[i + 1:]:
        if len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        try:
            v = float(d["Metric Value"].replace(",", ""))
        except ValueError:
            continue
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "ms": 1e-3,
                 "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3}.get(d["Metric Unit"], 1)
        e = by.setdefault(int(d["ID"]), {"name": d["Kernel Name"].split("(")[0][:40], "bytes": 0.0, "t": 0.0})
        if d["Metric Name"].startswith("dram__bytes"):
            e["bytes"] += v * scale
        else:
            e["t"] += v * scale
    return [by[k] for k in sorted(by)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cmd", choices=["run", "sum"])
    ap.add_argument("arg", nargs="?")
    ap.add_argument("--impl", default="merged", choices=["merged", "lbl"])
    ap.add_argument("--config", default="cfg2")
    a = ap.parse_args()
    if a.cmd == "run":
        run(a.impl, a.config)
    else:
        tot, per, n = summarize(a.arg)
        rd, wr = tot["dram__bytes_read.sum"], tot["dram__bytes_write.sum"]
        print(f"{os.path.basename(a.arg)}: {n} kernels, DRAM read {rd / 1e6:.1f} MB + write {wr / 1e6:.1f} MB = "
              f"{(rd + wr) / 1e6:.1f} MB, kernel time (cold, serialized) {tot['gpu__time_duration.sum'] * 1e3:.3f} ms")
        for k, v in sorted(per.items(), key=lambda kv: -(kv[1]["dram__bytes_read.sum"] + kv[1]["dram__bytes_write.sum"]))[:6]:
            print(f"    {k:40s} {(v['dram__bytes_read.sum'] + v['dram__bytes_write.sum']) / 1e6:10.1f} MB")
        if "merged" in os.path.basename(a.arg):   # one line per launch: brickify, each subgraph (+ pool tail), output
            for j, e in enumerate(per_launch(a.arg)):
                print(f"      launch {j:2d} {e['name']:40s} {e['bytes'] / 1e6:10.1f} MB")


if __name__ == "__main__":
    main()
