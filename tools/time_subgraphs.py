"""Per-subgraph device time of a configuration (CUDA events around each bdl_run_subgraph).

    python tools/time_subgraphs.py cfg3 [--mode memoized] [--reps 5]
"""
import argparse
import os
import sys

sys.path.insert(0, os.environ.get("BDL_ROOT") or os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--mode", default="auto")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--N", type=int, default=None)
    ap.add_argument("--max-layers", type=int, default=0)
    ap.add_argument("--fuse-pool", type=int, default=None)
    a = ap.parse_args()
    wl = workloads.make_workload(a.cfg, N=a.N)
    kw = {}
    if a.max_layers:
        kw["max_subgraph_layers"] = a.max_layers
    if a.fuse_pool is not None:
        kw["fuse_pool"] = a.fuse_pool
    plan = engine.plan_from_workload(wl, **kw)
    if a.mode != "auto":
        plan.set_mode(a.mode)
    xb = plan.brickify(wl["x"])
    yb = plan.alloc_bricked(plan.out_layout)
    for _ in range(2):
        plan.run(xb, yb)
    torch.cuda.synchronize()
    sgs = plan.subgraphs()
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(len(sgs) + 1)] for _ in range(a.reps)]
    for r in range(a.reps):
        ev[r][0].record()
        for i in range(len(sgs)):
            plan.run_subgraph(i, xb, yb)
            ev[r][i + 1].record()
    torch.cuda.synchronize()
    shapes = {-1: (wl["D"], wl["H"], wl["W"])}
    fl = []
    for j, l in enumerate(wl["layers"]):
        o = workloads.layer_out_shape(l, *shapes[l["input"]])
        shapes[j] = o
        fl.append(2 * wl["N"] * o[0] * o[1] * o[2] * l["cout"] * l["cin"] * l["k"][0] * l["k"][1] * l["k"][2]
                  if l["kind"] == "conv" else 0)
    tot = 0.0
    for i, s in enumerate(sgs):
        ms = sorted(ev[r][i].elapsed_time(ev[r][i + 1]) for r in range(a.reps))[a.reps // 2]
        tot += ms
        ls = wl["layers"][s["first"]:s["last"] + 1]
        desc = " ".join(f"{l['kind'][0]}{l['cin']}>{l['cout']}k{l['k'][-1]}s{l['stride'][-1]}" for l in ls)
        f = sum(fl[s["first"]:s["last"] + 1])
        print(f"{i:3d} [{s['first']:2d},{s['last']:2d}] {s['mode']:9s} {s['kernel']:16s} {ms:9.3f} ms "
              f"{f / ms / 1e9:7.1f} TF/s  {desc}")
    print(f"total {tot:.3f} ms")


if __name__ == "__main__":
    main()
