"""Debug helper: run each subgraph of a configuration with a device sync after it (several passes)."""
import sys

import torch

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads

cfg, N, fb = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
passes = int(sys.argv[4]) if len(sys.argv) > 4 else 1
only = int(sys.argv[5]) if len(sys.argv) > 5 else -1
wl = workloads.make_workload(cfg, N=N)
plan = engine.plan_from_workload(wl, force_brick=fb) if fb else engine.plan_from_workload(wl)
xb = plan.brickify(wl["x"])
yb = plan.alloc_bricked(plan.out_layout)
for r in range(passes):
    for i, s in enumerate(plan.subgraphs()):
        if only >= 0 and i != only:
            continue
        plan.run_subgraph(i, xb, yb)
        torch.cuda.synchronize()
        print("pass", r, "ok", i, s["mode"], s["kernel"], s["model_brick"], flush=True)
