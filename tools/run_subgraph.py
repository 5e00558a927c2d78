"""Run one subgraph of a configuration a few times (profiling helper: `ncu -k gen_kernel -s <n> -c 1` captures the
last launch).    python tools/run_subgraph.py cfg4 1 [mode]"""
import sys, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
cfg, i = sys.argv[1], int(sys.argv[2])
wl = workloads.make_workload(cfg)
plan = engine.plan_from_workload(wl)
if len(sys.argv) > 3:
    plan.set_mode(sys.argv[3])
xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
plan.run(xb, yb)
for _ in range(2):
    plan.run_subgraph(i, xb, yb)
torch.cuda.synchronize()
