"""A/B whole-config subgraph time of another checkout: python tools/ab_sub.py <repo root> <cfg> [mode]"""
import os, sys
root = os.path.abspath(sys.argv[1])
sys.path.insert(0, root)
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
wl = workloads.make_workload(sys.argv[2])
plan = engine.plan_from_workload(wl)
if len(sys.argv) > 3: plan.set_mode(sys.argv[3])
xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
for _ in range(3): plan.run(xb, yb)
ts = []
for _ in range(7):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); plan.run(xb, yb); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
ts.sort()
print(f"{os.path.basename(root):6s} {sys.argv[2]} {sys.argv[3] if len(sys.argv) > 3 else 'auto'} median {ts[3]:.3f} ms")
