"""B200 re-run of the paper's two microbenchmark sweeps (§4.6, Figs 10-11).

  Fig 10 analogue: a 6-layer 3x3x3 chain, 64 channels, stride 1, no padding, on a 112^3
                   volume, partitioned 1+1+1+1+1+1 / 2+2+2 / 3+3 / 6 (max_subgraph_layers), modes
                   memoized / padded / the model's choice.
  Fig 11 analogue: a 3-layer chain of the same layers on 224^3 (or --big), brick edge 4 / 8 / 16 / 32.

Prints one line per point: partition or brick, mode, device time (CUDA events around bdl_run after warm-up),
useful TFLOP/s.  Synthetic seeded data (workloads.make_graph_workload); run on one B200:
    python tools/sweep_fig10_11.py [--d10 112] [--d11 224]
"""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads as W


def chain(n, C):
    return [W.conv(C, C, 3, 1, 0, nsp=3) for _ in range(n)]


def flops(layers, D):
    f, d = 0, D
    for l in layers:
        d = d - 2
        f += 2 * d ** 3 * l["cout"] * l["cin"] * 27
    return f


def timeit(plan, xb, yb, reps=5):
    for _ in range(2):
        plan.run(xb, yb)
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); plan.run(xb, yb); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
    return sorted(ts)[reps // 2]


def point(layers, D, C, brick, mode, **opt):
    wl = W.make_graph_workload(layers, 1, C, D, D, D, 3, brick, "bf16", seed=77)
    plan = engine.plan_from_workload(wl, **opt)
    if mode != "auto":
        plan.set_mode(mode)
    sgs = plan.subgraphs()
    xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
    ms = timeit(plan, xb, yb)
    part = "+".join(str(s["last"] - s["first"] + 1) for s in sgs)
    modes = "/".join(sorted({s["mode"] for s in sgs}))
    return ms, part, modes, sgs


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--d10", type=int, default=112)
    ap.add_argument("--d11", type=int, default=224)
    ap.add_argument("--C", type=int, default=64)
    a = ap.parse_args()
    C = a.C
    L6 = chain(6, C)
    f6 = flops(L6, a.d10)
    print(f"# Fig 10 analogue: 6 x conv3^3 (valid), C={C}, {a.d10}^3, 8^3 bricks")
    for maxl in (1, 2, 3, 6):
        for mode in ("auto", "memoized", "padded"):
            if maxl == 1 and mode != "auto":
                continue
            try:
                ms, part, modes, sgs = point(L6, a.d10, C, (1, 8, 8, 8), mode, max_subgraph_layers=maxl,
                                              onchip_budget=1 << 36)
                print(f"  partition {part:12s} mode {modes:22s} {ms:8.3f} ms  {f6 / ms / 1e9:7.1f} TF/s  "
                      f"delta {[round(s['delta'], 3) for s in sgs]}")
            except Exception as e:  # noqa: BLE001
                print(f"  max_layers {maxl} mode {mode}: {e}")
    L3 = chain(3, C)
    f3 = flops(L3, a.d11)
    print(f"# Fig 11 analogue: 3 x conv3^3 (valid), C={C}, {a.d11}^3, brick edge sweep")
    for b in (4, 8, 16, 32):
        for mode in ("auto", "memoized"):
            try:
                ms, part, modes, sgs = point(L3, a.d11, C, (1, b, b, b), mode, force_brick=b)
                print(f"  brick {b:2d}^3 partition {part:6s} mode {modes:22s} {ms:8.3f} ms  {f3 / ms / 1e9:7.1f} TF/s")
            except Exception as e:  # noqa: BLE001
                print(f"  brick {b}: {e}")
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
