"""Benchmark: merged conv-chain inference throughput (images/s) on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config cfg2] [--mode auto|padded|memoized|unmerged]
    python bench.py --impl reference ...        # the CPU oracle arm (tier rule: the reference arm is the oracle)

Workload (BASELINE.json configs[1]): ResNet-18 conv2_x basic block, bf16, N=64 per GPU, 56x56x64,
8x8 bricks; one step = brickify (dense NCHW -> bricks) + every merged subgraph of the plan
(static-analysis mode choice) + unbrickify, inputs resident in HBM.  L2 is flushed (256 MiB
write) between timed steps, outside the timed events.  Multi-GPU: one process per GPU (torchrun),
each rank runs its own 64-image shard ("weak" scaling, no data-path collective); the timed region
is bracketed by barrier + synchronize, and the time is the max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_PEAKS = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--config", default="cfg2")
    ap.add_argument("--mode", default="auto")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cudnn", action="store_true")
    ap.add_argument("--no-extra", action="store_true",
                    help="skip the other configurations (cfg3/cfg4/cfg5 and cfg2 padded) measured in the default run")
    ap.add_argument("--micro", type=int, default=2, help="strong scaling: micro-batches per rank for the gather overlap")
    ap.add_argument("--strong", action="store_true",
                    help="strong scaling with the overlapped output gather (default for cfg4 when WORLD_SIZE > 1)")
    ap.add_argument("--spatial", action="store_true",
                    help="3-D configs: shard ONE volume into depth slabs with a brick-plane halo exchange "
                         "(default for 3-D configs when WORLD_SIZE > 1)")
    return ap.parse_args()


def load_peaks():
    try:
        with open(PEAKS_PATH) as f:
            p = json.load(f)
        return p, "measured"
    except Exception:
        return dict(FALLBACK_PEAKS), "fallback"


def workload_desc(wl):
    return (f"{wl['cfg']}: ResNet-18 conv2_x basic block (conv3x3+b+ReLU -> conv3x3+b, +x, ReLU), "
            f"N={wl['N']} C={wl['C']} {wl['H']}x{wl['W']}, {wl['brick'][2]}x{wl['brick'][3]} bricks"
            if wl["cfg"] == "cfg2" else f"{wl['cfg']} N={wl['N']} C={wl['C']} D={wl['D']} H={wl['H']} W={wl['W']}")


def useful_flops(wl):
    """2*MACs of plain layer-by-layer execution (padded-mode recompute not credited).  Each layer's
    input extent is that of the layer it reads (`input`), so branches (projections) are sized right."""
    from paper_conf_icpp_lakshminarasimhan24_b200 import workloads
    f = 0
    shapes = {-1: (wl["D"], wl["H"], wl["W"])}
    for i, l in enumerate(wl["layers"]):
        D, H, W = shapes[l["input"]]
        Do, Ho, Wo = workloads.layer_out_shape(l, D, H, W)
        if l["kind"] == "conv":
            kd, kh, kw = l["k"]
            f += 2 * wl["N"] * Do * Ho * Wo * l["cout"] * l["cin"] * kd * kh * kw
        shapes[i] = (Do, Ho, Wo)
    return f


def subgraph_roofline(wl, sgs, peak_tflops, hbm_gbs):
    """t_roof = sum over subgraphs of max(F_s / P_tensor, Bytes_s / HBM).  F_s = useful conv FLOPs
    (2*MACs of layer-by-layer execution; padded recompute not credited); Bytes_s = algorithmic merged bytes: every
    tensor the subgraph reads from outside (its input, external residuals / branch inputs) once, every tensor it
    leaves for later subgraphs (its output, inner live-outs) once, its weights once (bf16 storage)."""
    from paper_conf_icpp_lakshminarasimhan24_b200 import workloads
    L = wl["layers"]
    esz = 2 if wl["dtype"] == "bf16" else 4
    shapes = {-1: (wl["D"], wl["H"], wl["W"])}
    chans = {-1: wl["C"]}
    flops = []
    for i, l in enumerate(L):
        D, H, W = shapes[l["input"]]
        o = workloads.layer_out_shape(l, D, H, W)
        shapes[i], chans[i] = o, l["cout"]
        flops.append(2 * wl["N"] * o[0] * o[1] * o[2] * l["cout"] * l["cin"] * l["k"][0] * l["k"][1] * l["k"][2]
                     if l["kind"] == "conv" else 0)
    tb = lambda m: wl["N"] * chans[m] * shapes[m][0] * shapes[m][1] * shapes[m][2] * esz   # noqa: E731
    t_roof, per = 0.0, []
    for s in sgs:
        f, e = s["first"], s["last"]
        reads = set()
        for j in range(f, e + 1):
            for m in (L[j]["input"], L[j]["residual"]):
                if m is not None and m < f:
                    reads.add(m)
        writes = {e} | {j for j in range(f, e) if any(L[m]["input"] == j or L[m]["residual"] == j
                                                      for m in range(e + 1, len(L)))}
        wbytes = sum(L[j]["cout"] * L[j]["cin"] * L[j]["k"][0] * L[j]["k"][1] * L[j]["k"][2] * esz
                     for j in range(f, e + 1) if L[j]["kind"] == "conv")
        F = sum(flops[f:e + 1])
        B = sum(tb(m) for m in reads) + sum(tb(m) for m in writes) + wbytes
        t = max(F / (peak_tflops * 1e12), B / (hbm_gbs * 1e9))
        t_roof += t
        per.append({"layers": [f, e], "gflop": F / 1e9, "mbytes": B / 1e6, "t_roof_ms": t * 1e3})
    return t_roof * 1e3, per


def measure_config(cfg, dev, K, flush, peaks, mode=None, cudnn=True):
    """One more configuration measured in the same run (same contract as the headline: K steps of brickify +
    merged subgraphs + unbrickify with inputs resident in HBM, L2 flushed between steps, events around each step;
    a second pass with events around each subgraph for the per-subgraph times)."""
    import torch
    from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
    wl = workloads.make_workload(cfg)
    plan = engine.plan_from_workload(wl, device=dev)
    if mode:
        plan.set_mode(mode)
    sgs = plan.subgraphs()
    x = wl["x"].to(device=dev, dtype=plan.tdtype).contiguous()
    xb = plan.alloc_bricked(plan.in_layout)
    yb = plan.alloc_bricked(plan.out_layout)
    lo = plan.out_layout
    y = torch.empty((lo.N, lo.C, lo.D, lo.H, lo.W), dtype=plan.tdtype, device=dev)
    for _ in range(3):
        plan.forward_into(x, y)
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for a, b in ev:
        flush()
        a.record()
        plan.brickify(x, out=xb)
        plan.run_dense(xb, out=y)
        b.record()
    torch.cuda.synchronize()
    step_ms = statistics.mean(a.elapsed_time(b) for a, b in ev)
    sev = [[torch.cuda.Event(enable_timing=True) for _ in range(len(sgs) + 1)] for _ in range(K)]
    for e in sev:
        flush()
        plan.brickify(x, out=xb)
        e[0].record()
        for i in range(len(sgs)):
            plan.run_subgraph(i, xb, yb)
            e[i + 1].record()
    torch.cuda.synchronize()
    sub_ms = [statistics.median(e[i].elapsed_time(e[i + 1]) for e in sev) for i in range(len(sgs))]
    peak = float(peaks["bf16_tflops"]) if wl["dtype"] == "bf16" else None
    out = {"workload": workload_desc(wl), "mode": "/".join(sorted({g["mode"] for g in sgs})),
           "subgraphs": len(sgs), "ms_per_step": step_ms, "images_per_s": wl["N"] / (step_ms / 1e3),
           "merged_ms": sum(sub_ms), "gpu_launches_per_step": 2 + plan.launches_per_run}
    if peak:
        flops = useful_flops(wl)
        t_roof, per = subgraph_roofline(wl, sgs, peak, float(peaks["hbm_gbs"]))
        out["roofline"] = {"t_roof_ms": t_roof, "frac_merged": t_roof / sum(sub_ms), "frac_step": t_roof / step_ms,
                           "useful_tflops_merged": flops / (sum(sub_ms) / 1e3) / 1e12, "peak_tflops": peak,
                           "how": "t_roof = sum_s max(F_s/P_bf16, Bytes_s/HBM) (SURVEY 8(d)); frac = t_roof / measured"}
        out["per_subgraph"] = [dict(p, ms=m, mode=g["mode"], kernel=g["kernel"])
                               for p, m, g in zip(per, sub_ms, sgs)]
    if cudnn:
        out["cudnn_layer_by_layer"] = cudnn_lbl(wl, dev, K, flush)
    del plan, xb, yb, x, y
    torch.cuda.empty_cache()
    return out


# ------------------------------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index=0):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 8:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for nm, v in zip(names, r[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


# ------------------------------------------------------------------------------------------ oracle arms
def oracle_images_per_s(wl, n_images, threads):
    import oracle
    os.environ["OMP_NUM_THREADS"] = str(threads)
    x = wl["x"].numpy()[:n_images]
    t = time.perf_counter()
    oracle.run_graph(wl["layers"], x, wl["weights"], wl["biases"], dtype=wl["dtype"])
    return n_images / (time.perf_counter() - t)


def cpu_baseline(wl, budget_s=12.0):
    """The oracle as it stands, on this host's cores, on a bounded sample of the same workload."""
    import oracle
    threads = os.cpu_count() or 1
    os.environ["OMP_NUM_THREADS"] = str(threads)
    oracle.lib()
    x = wl["x"].numpy()
    t = time.perf_counter()
    oracle.run_graph(wl["layers"], x[:1], wl["weights"], wl["biases"], dtype=wl["dtype"])
    t1 = time.perf_counter() - t
    n = int(max(1, min(wl["N"], budget_s / max(t1, 1e-3))))
    ips = oracle_images_per_s(wl, n, threads)
    return {"value": ips, "unit": "images/s", "cores": threads, "kind": "oracle",
            "sample": f"{n} of {wl['N']} images of the same workload, fp64 direct conv, OpenMP {threads} threads"}


def run_reference(args):
    from paper_conf_icpp_lakshminarasimhan24_b200 import workloads
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    wl = workloads.make_workload(args.config)
    import oracle
    threads = os.cpu_count() or 1
    os.environ["OMP_NUM_THREADS"] = str(threads)
    oracle.lib()
    per_step = 4  # images per step: a bounded sample of the workload
    x = wl["x"].numpy()
    for _ in range(args.warmup):
        oracle.run_graph(wl["layers"], x[:per_step], wl["weights"], wl["biases"], dtype=wl["dtype"])
    t = time.perf_counter()
    for s in range(args.steps):
        i0 = (s * per_step) % wl["N"]
        oracle.run_graph(wl["layers"], x[i0:i0 + per_step], wl["weights"], wl["biases"], dtype=wl["dtype"])
    dt = time.perf_counter() - t
    v = per_step * args.steps / dt
    line = {"impl": "reference", "metric": "images/sec merged conv chain per B200", "value": v, "unit": "images/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_desc(wl), "sample_per_step": f"{per_step} of {wl['N']} images"},
            "cpu_baseline": {"value": v, "unit": "images/s", "cores": threads, "kind": "oracle",
                             "sample": f"{per_step} images per step x {args.steps} steps"},
            "e2e": {"value": v, "unit": "images/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


# ------------------------------------------------------------------------------------------ native arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)

    if workloads.CONFIGS[args.config]["nsp"] == 3 and (world > 1 or args.spatial):
        return bench_spatial(args, world, rank, local, dev)
    if args.strong or (args.config == "cfg4" and world > 1):
        return bench_strong(args, world, rank, local, dev)
    wl = workloads.make_workload(args.config, input_seed_offset=rank)
    plan = engine.plan_from_workload(wl, device=dev)
    if args.mode != "auto":
        plan.set_mode(args.mode)
    sg = plan.subgraphs()
    stream = torch.cuda.current_stream(dev)

    x_dense = wl["x"].to(device=dev, dtype=plan.tdtype).contiguous()
    xb = plan.alloc_bricked(plan.in_layout)
    yb = plan.alloc_bricked(plan.out_layout)
    y_dense = torch.empty((plan.out_layout.N, plan.out_layout.C, plan.out_layout.D, plan.out_layout.H,
                           plan.out_layout.W), dtype=plan.tdtype, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    flush_rd = torch.ones(64 << 20, dtype=torch.float32, device=dev)   # 256 MiB

    def flush_l2():
        # write a buffer larger than L2, then stream-read another one so the dirty flush lines are written
        # back now (outside the timed events) instead of inside the first timed kernel
        flush.zero_()
        flush_rd.sum()

    def step():
        plan.brickify(x_dense, out=xb)
        plan.run_dense(xb, out=y_dense)

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()

    K = args.steps
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(K)]
    sv = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(K)]
    with ClockSampler(local) as clk:
        # keep the GPU loaded (untimed) while the clock sampler starts, so that its samples cover the
        # timed region under load
        t_end = time.time() + 0.5
        while time.time() < t_end:
            for _ in range(20):
                step()
            torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        # (1) the K timed steps: events only around each step.  An event recorded between two kernels
        #     would stop the next kernel's programmatic-dependent launch from overlapping the previous
        #     one's tail (measured: +8 us per cfg2 step), so the step is timed as the user runs it.
        for k in range(K):
            flush_l2()                         # L2 flush, outside the timed events
            sv[k][0].record(stream)
            plan.brickify(x_dense, out=xb)
            plan.run_dense(xb, out=y_dense)   # merged subgraphs, unbrickify fused into the last epilogue
            sv[k][1].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        # (2) K more steps with events between the kernels: per-kernel breakdown and the roofline's
        #     kernel duration (each kernel then runs without overlap, which is what its roofline needs)
        for k in range(K):
            flush_l2()
            e = ev[k]
            e[0].record(stream)
            plan.brickify(x_dense, out=xb)
            e[1].record(stream)
            plan.run_dense(xb, out=y_dense)    # the merged subgraph launch(es) of the step: roofline kernel time
            e[2].record(stream)
            plan.run(xb, yb)                   # (breakdown only) bricked-output run + separate unbrickify
            e[3].record(stream)
            plan.unbrickify(yb, out=y_dense)
            e[4].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [e[0].elapsed_time(e[1]) for e in sv]
    run_ms = [e[1].elapsed_time(e[2]) for e in ev]
    total_ms = sum(step_ms)
    t_local = torch.tensor([total_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t_local, op=dist.ReduceOp.MAX)
    total_ms = float(t_local.item())
    images = wl["N"] * world * K
    value = images / (total_ms / 1e3)

    # ---- end to end through the public API: pinned host input -> device -> ... -> pinned host output
    x_host = wl["x"].to(plan.tdtype).contiguous().pin_memory()
    y_host = torch.empty(y_dense.shape, dtype=plan.tdtype).pin_memory()
    x_dev2 = torch.empty_like(x_dense)
    for _ in range(3):
        x_dev2.copy_(x_host, non_blocking=True)
        plan.unbrickify(plan.run(plan.brickify(x_dev2, out=xb), yb), out=y_dense)
        y_host.copy_(y_dense, non_blocking=True)
    torch.cuda.synchronize()
    e2e_ms = 0.0
    for k in range(K):
        flush_l2()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        x_dev2.copy_(x_host, non_blocking=True)
        plan.brickify(x_dev2, out=xb)
        plan.run_dense(xb, out=y_dense)
        y_host.copy_(y_dense, non_blocking=True)
        b.record(stream)
        b.synchronize()
        e2e_ms += a.elapsed_time(b)
    t2 = torch.tensor([e2e_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t2, op=dist.ReduceOp.MAX)
    e2e_serial = images / (float(t2.item()) / 1e3)
    e2e_pipe_ms = e2e_pipelined(plan, wl, x_dense, y_dense, xb, yb, K, dev)
    t3 = torch.tensor([e2e_pipe_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t3, op=dist.ReduceOp.MAX)
    e2e_value = images / (float(t3.item()) / 1e3)

    # ---- roofline of the dominant kernel (the merged subgraph launch)
    peaks, peak_src = load_peaks()
    flops = useful_flops(wl)
    kernel_ms = statistics.mean(run_ms)
    traffic, traffic_src = None, None
    tp = os.path.join(ROOT, "profiles", "ncu_summary_latest.json")
    if os.path.exists(tp):
        try:
            with open(tp) as f:
                traffic = json.load(f).get("dram_bytes_per_launch", {}).get(sg[0]["kernel"])
            traffic_src = ("file lookup, not measured in this run: dram__bytes_read.sum + dram__bytes_write.sum of one "
                           "launch from the committed ncu --set full capture summarised in profiles/ncu_summary_latest.json")
        except Exception:
            traffic = None
    kinds = {g["kernel"] for g in sg}
    if kinds == {"cuda-core brick"}:
        # plain FMA pipes: measured on this box (8 independent FFMA chains per thread, 4 x 256 threads per SM;
        # libbdl_microbench.so), the derived figure 148 SM x 128 FFMA/clk x 2 x 1965 MHz as a fallback
        bound = "alu"
        try:
            import ctypes
            from paper_conf_icpp_lakshminarasimhan24_b200 import build as _b
            mb = ctypes.CDLL(_b.build_microbench())
            tf = ctypes.c_double()
            if mb.bdl_mb_ffma(ctypes.byref(tf)) != 0:
                raise RuntimeError("ffma microbenchmark failed")
            peak, peak_src = tf.value, "measured in this run: FFMA microbenchmark (libbdl_microbench.so bdl_mb_ffma)"
        except Exception as e:
            peak = 148 * 128 * 2 * 1.965e9 / 1e12
            peak_src = f"derived (microbenchmark unavailable: {e}): 148 SM x 128 FFMA/clk x 2 x 1965 MHz"
    else:
        bound, peak = "tensor", float(peaks["bf16_tflops"])
        peak_src = f"{peak_src} bf16_tflops (burst, cuBLAS 8192^3)"
    achieved = flops / (kernel_ms / 1e3) / 1e12
    kname = sg[0]["kernel"] if len(sg) == 1 else f"{len(sg)} subgraph launches ({', '.join(sorted(kinds))})"
    if len(sg) == 1 and sg[0].get("cta_pair") and sg[0]["mode"] != "padded":
        kname += ", CTA pair (cta_group::2, memo_pair_kernel)"
    roofline = {"bound": bound, "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                "traffic": traffic if len(sg) == 1 and kinds == {"tcgen05 band"} else None,
                "traffic_source": traffic_src if len(sg) == 1 and kinds == {"tcgen05 band"} else None,
                "peak_source": peak_src,
                "kernel": f"{kname} ({'/'.join(sorted({g['mode'] for g in sg}))})",
                "algorithmic_flops_per_launch": flops, "kernel_ms_mean": kernel_ms, "hbm_frac_of_step_bytes": None}
    # step bytes
    in_b = x_dense.numel() * x_dense.element_size()
    out_b = y_dense.numel() * y_dense.element_size()
    step_bytes = 3 * in_b + out_b   # brickify (read + write), merged (read bricks, write the dense output)
    roofline["hbm_frac_of_step_bytes"] = step_bytes / (statistics.mean(step_ms) / 1e3) / 1e9 / float(peaks["hbm_gbs"])

    # ---- layer-by-layer cuDNN reference (context): torch conv2d, channels_last bf16
    cudnn = None
    if not args.no_cudnn and rank == 0:
        cudnn = cudnn_lbl(wl, dev, K, flush_l2)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(wl)

    # ---- the other configurations, in the same run (driver-observed): cfg2 padded mode, cfg3, cfg4, cfg5
    extra = None
    if rank == 0 and world == 1 and not args.no_extra and args.config == "cfg2" and args.mode == "auto":
        extra = {}
        del xb, yb
        torch.cuda.empty_cache()
        Ke = max(3, min(K, 10))
        for name, cfg, mode in (("cfg2_padded", "cfg2", "padded"), ("cfg3", "cfg3", None), ("cfg4", "cfg4", None),
                                ("cfg5", "cfg5", None)):
            try:
                extra[name] = measure_config(cfg, dev, Ke, flush_l2, load_peaks()[0], mode=mode,
                                             cudnn=not args.no_cudnn and name != "cfg2_padded")
            except Exception as e:   # report, do not hide: the headline line still prints
                extra[name] = {"error": f"{type(e).__name__}: {str(e)[:300]}"}

    if rank == 0:
        launches = K * (1 + plan.launches_per_run)   # brickify + the merged launches (unbrickify fused)
        line = {
            "metric": "images/sec merged conv chain per B200", "value": value, "unit": "images/s",
            "n_gpus": world, "steps": K, "warmup": max(3, args.warmup), "ms_per_step": total_ms / K,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": wl["dtype"],
            "data": "synthetic (seeded N(0,1) inputs, He-normal weights; workloads.py)",
            "config": {"workload": workload_desc(wl), "images_per_gpu": wl["N"], "global_batch": wl["N"] * world,
                       "mode": sg[0]["mode"], "mode_model": sg[0]["mode_model"], "delta": round(sg[0]["delta"], 4),
                       "kernel": sg[0]["kernel"] + (", CTA pair (cta_group::2)" if sg[0].get("cta_pair") else ""),
                       "subgraphs": len(sg), "step": "brickify + merged subgraph with unbrickify fused into its last epilogue (bdl_run_dense)",
                       "l2": "flushed between timed steps (256 MiB write + 256 MiB read, outside the events)",
                       "timing": "value/ms_per_step: K steps with events only around each step; breakdown_ms and "
                                 "roofline: a second K-step pass with events between the kernels",
                       "parallelism": f"batch-sharded x{world}, no data-path collective"},
            "clocks": clk.summary(),
            "e2e": {"value": e2e_value, "unit": "images/s", "h2d_bytes_per_step": x_host.numel() * x_host.element_size(),
                    "d2h_bytes_per_step": y_host.numel() * y_host.element_size(),
                    "how": "public serving API engine.HostPipeline on pinned HOST buffers: every step copies its "
                           "input H2D and its output D2H inside the timed region; steps pipelined over three buffer "
                           "slots on three streams (H2D of step k+1 and D2H of step k-1 overlap step k); last output "
                           "checked bit-exact against the device path; no L2 flush (inputs arrive over PCIe)",
                    "serial_value": e2e_serial},
            "gpu_launches": launches,
            "roofline": roofline,
            "cpu_baseline": cpu,
            "breakdown_ms": {"brickify": statistics.mean(e[0].elapsed_time(e[1]) for e in ev),
                             "merged_subgraph_dense_out": kernel_ms,
                             "merged_subgraph_bricked_out": statistics.mean(e[2].elapsed_time(e[3]) for e in ev),
                             "separate_unbrickify": statistics.mean(e[3].elapsed_time(e[4]) for e in ev),
                             "step_with_events_between_kernels": statistics.mean(e[0].elapsed_time(e[2]) for e in ev)},
            "cudnn_layer_by_layer": cudnn,
            "other_configs": extra,
        }
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()
    return 0


def e2e_pipelined(plan, wl, x_dense, y_dense, xb, yb, K, dev):
    """End-to-end time (ms) of K requests through the public serving API (engine.HostPipeline): pinned
    HOST input -> H2D -> brickify -> merged subgraphs -> unbrickify -> D2H -> host, consecutive requests
    overlapped on three streams.  The last output is checked bit for bit against the device-timed path."""
    import torch
    from paper_conf_icpp_lakshminarasimhan24_b200 import engine
    pipe = engine.HostPipeline(plan, slots=3)
    x_host = wl["x"].to(plan.tdtype).contiguous().pin_memory()
    pipe.run([x_host] * 4)
    torch.cuda.synchronize(dev)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(pipe.s_h2d)
    pipe.s_cmp.wait_event(a)
    pipe.s_d2h.wait_event(a)
    pipe.run([x_host] * K, on_output=lambda k, y: None)
    # (the callbacks drain D2H completions on the host; the device end is the last D2H)
    pipe.s_h2d.wait_stream(pipe.s_cmp)
    pipe.s_h2d.wait_stream(pipe.s_d2h)
    b.record(pipe.s_h2d)
    b.synchronize()
    ms = a.elapsed_time(b)
    plan.run_dense(plan.brickify(x_dense, out=xb), out=y_dense)
    torch.cuda.synchronize(dev)
    if not torch.equal(pipe.y_host[(K - 1) % pipe.slots], y_dense.cpu()):
        raise RuntimeError("pipelined e2e output differs from the device-timed path")
    return ms


def bench_spatial(args, world, rank, local, dev):
    """One 3-D volume split into `world` depth slabs (strong scaling): per step each rank brickifies its slab
    into an extended buffer, exchanges one brick plane of halo per face with its neighbours (NCCL
    point-to-point over NVLink), runs the merged plan on the extended slab and unbrickifies its own planes."""
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_lakshminarasimhan24_b200 import parallel, workloads
    wl = workloads.make_workload(args.config)
    run = parallel.SpatialRunner(wl["layers"], wl["weights"], wl["biases"], wl["C"], wl["D"], wl["H"], wl["W"],
                                 wl["brick"], wl["dtype"], rank, world, device=dev,
                                 mode=None if args.mode == "auto" else args.mode)
    g = run.geo
    x_own = wl["x"][:, :, g.lo:g.hi].to(device=dev, dtype=run.plan.tdtype).contiguous()
    y_own = torch.empty((1, run.own_out.C, g.own, wl["H"], wl["W"]), dtype=run.plan.tdtype, device=dev)
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    flush_rd = torch.ones(64 << 20, dtype=torch.float32, device=dev)
    exch = run.exchange if world > 1 else (lambda: None)

    def step():
        run.load(x_own)
        exch()
        run.compute(out=y_own)

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()
    K = args.steps
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(K)]
    with ClockSampler(local) as clk:
        t_end = time.time() + 0.5
        while time.time() < t_end:
            for _ in range(5):
                step()
            torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        for k in range(K):
            flush.zero_()
            flush_rd.sum()
            if world > 1:
                dist.barrier()
            e = ev[k]
            e[0].record(stream)
            run.load(x_own)
            exch()
            e[1].record(stream)
            run.plan.run(run.xb, run.yb)
            e[2].record(stream)
            run.plan.unbrickify(run.yb[g.own_slice(run.out_plane)], layout=run.own_out, out=y_own)
            e[3].record(stream)
        torch.cuda.synchronize()
    step_ms = [e[0].elapsed_time(e[3]) for e in ev]
    t = torch.tensor([sum(step_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_ms = float(t.item())
    kernel_ms = statistics.mean(e[1].elapsed_time(e[2]) for e in ev)
    flops = useful_flops(wl)
    peaks, peak_src = load_peaks()
    achieved = flops / world / (kernel_ms / 1e3) / 1e12
    if rank == 0:
        line = {
            "metric": "images/sec merged conv chain per B200", "value": K / (total_ms / 1e3), "unit": "volumes/s",
            "n_gpus": world, "steps": K, "warmup": max(3, args.warmup), "ms_per_step": total_ms / K,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": wl["dtype"],
            "data": "synthetic (seeded N(0,1) inputs, He-normal weights; workloads.py)",
            "config": {"workload": workload_desc(wl), "global_batch": 1,
                       "parallelism": f"spatial depth slabs x{world}, {g.halo_planes}-brick-plane halo exchange "
                                      f"(NCCL point-to-point)",
                       "slab_planes": g.own, "halo_planes_per_face": g.halo_planes * wl["brick"][1],
                       "mode": run.plan.subgraphs()[0]["mode"],
                       "l2": "flushed between timed steps (256 MiB write + 256 MiB read, outside the events)"},
            "clocks": clk.summary(),
            "gpu_launches": K * (2 + run.plan.launches_per_run),
            "roofline": {"bound": "tensor", "achieved": achieved, "peak": float(peaks["bf16_tflops"]),
                         "unit": "TFLOP/s", "frac": achieved / float(peaks["bf16_tflops"]), "traffic": None,
                         "peak_source": f"{peak_src} bf16_tflops",
                         "kernel": "merged subgraph on the extended slab (useful FLOPs of the own slab)"},
            "breakdown_ms": {"brickify+halo_exchange": statistics.mean(e[0].elapsed_time(e[1]) for e in ev),
                             "merged_subgraph": kernel_ms,
                             "unbrickify": statistics.mean(e[2].elapsed_time(e[3]) for e in ev)},
        }
        print(json.dumps(line))
    if world > 1:
        dist.destroy_process_group()
    return 0


def bench_strong(args, world, rank, local, dev):
    """Strong scaling: the global batch of 256 images is split over the ranks in
    micro-batches; each rank runs brickify + merged subgraphs + unbrickify per micro-batch and all-gathers the
    outputs over NCCL on a communication stream while its next micro-batch computes (parallel.BatchRunner).  value =
    global images / max-over-ranks step time with the gather; sharded_value = the same with outputs left sharded."""
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_lakshminarasimhan24_b200 import engine, parallel, workloads
    if not dist.is_initialized():   # --strong at N = 1 without torchrun: a one-rank NCCL group (the same code path)
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    full = workloads.make_workload(args.config)
    n_total = full["N"]
    mb, ranges = parallel.micro_batches(n_total, world, args.micro)
    wl = workloads.make_workload(args.config, N=mb)
    plan = engine.plan_from_workload(wl, device=dev)
    if args.mode != "auto":
        plan.set_mode(args.mode)
    lo = plan.out_layout
    run = parallel.BatchRunner(n_total, (lo.C, lo.D, lo.H, lo.W), rank, world, micro=args.micro, plan=plan, device=dev)
    x_local = full["x"][run.global_images()].to(device=dev, dtype=plan.tdtype).contiguous()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    for _ in range(max(3, args.warmup)):
        run.forward(x_local)
    torch.cuda.synchronize()
    K = args.steps
    res = {}
    with ClockSampler(local) as clk:
        for gather in (True, False):
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
            dist.barrier()
            torch.cuda.synchronize()
            for a, b in ev:
                flush.zero_()
                a.record()
                run.forward(x_local, gather=gather)
                b.record()
            torch.cuda.synchronize()
            dist.barrier()
            t = torch.tensor([sum(a.elapsed_time(b) for a, b in ev)], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            res[gather] = float(t.item())
    # correctness of the gathered batch: this rank's own images equal its local results
    y = run.forward(x_local)
    mine = y[run.global_images()]
    ok = bool(torch.equal(mine, run.forward(x_local, gather=False)))
    peaks, peak_src = load_peaks()
    if rank == 0:
        line = {
            "metric": "images/sec merged conv chain per B200", "value": n_total * K / (res[True] / 1e3),
            "unit": "images/s", "n_gpus": world, "steps": K, "warmup": max(3, args.warmup),
            "ms_per_step": res[True] / K, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": wl["dtype"], "data": "synthetic (seeded N(0,1) inputs, He-normal weights; workloads.py)",
            "config": {"workload": workload_desc(full), "global_batch": n_total, "images_per_gpu": n_total // world,
                       "micro_batches": args.micro, "micro_batch": mb,
                       "parallelism": f"batch-sharded x{world}, outputs all-gathered (NCCL all_gather_into_tensor on a "
                                      f"comm stream, overlapped with the next micro-batch)",
                       "l2": "flushed between timed steps (256 MiB write, outside the events)"},
            "sharded_value": n_total * K / (res[False] / 1e3),
            "gather_check": ok,
            "clocks": clk.summary(),
            "gpu_launches": K * args.micro * (2 + plan.launches_per_run),
        }
        print(json.dumps(line))
    dist.destroy_process_group()
    return 0


def cudnn_lbl(wl, dev, K, flush):
    """Layer-by-layer torch/cuDNN run of the same graph (context only, not our product)."""
    import torch
    import torch.nn.functional as F
    try:
        nsp3 = wl["nsp"] == 3
        fmt = torch.channels_last_3d if nsp3 else torch.channels_last
        x = wl["x"] if nsp3 else wl["x"][:, :, 0]
        x = x.to(device=dev, dtype=torch.bfloat16).contiguous(memory_format=fmt)
        ws = [None if w is None else (w if nsp3 else w[:, :, 0]).to(device=dev, dtype=torch.bfloat16)
              .contiguous(memory_format=fmt) for w in wl["weights"]]
        bs = [None if b is None else b.to(device=dev, dtype=torch.bfloat16) for b in wl["biases"]]
        sl = slice(None) if nsp3 else slice(1, None)

        def fwd():
            outs = []
            for l, w, b in zip(wl["layers"], ws, bs):
                src = x if l["input"] == -1 else outs[l["input"]]
                if l["kind"] == "maxpool":
                    pool = F.max_pool3d if nsp3 else F.max_pool2d
                    y = pool(src, l["k"][sl], l["stride"][sl], l["pad"][sl])
                else:
                    conv = F.conv3d if nsp3 else F.conv2d
                    y = conv(src, w, b, stride=l["stride"][sl], padding=l["pad"][sl])
                if l["residual"] is not None:
                    y = y + (x if l["residual"] == -1 else outs[l["residual"]])
                if l["relu"]:
                    y = torch.relu(y)
                outs.append(y)
            return outs[-1]
        with torch.no_grad():
            for _ in range(5):
                fwd()
            torch.cuda.synchronize()
            tot = 0.0
            for _ in range(K):
                flush()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                fwd()
                b.record()
                b.synchronize()
                tot += a.elapsed_time(b)
        return {"ms_per_step": tot / K, "images_per_s": wl["N"] * K / (tot / 1e3),
                "what": "torch conv (cuDNN) bf16 channels_last, separate add/ReLU/pool, dense channels-last in/out"}
    except Exception as e:  # context measurement only
        return {"error": str(e)[:200]}


if __name__ == "__main__":
    sys.exit(main())
