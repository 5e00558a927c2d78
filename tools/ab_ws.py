"""A/B the cfg2 merged kernel of another checkout: python tools/ab_ws.py <repo root>"""
import os, sys
root = os.path.abspath(sys.argv[1])
sys.path.insert(0, root)
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
import paper_conf_icpp_lakshminarasimhan24_b200 as pkg
wl = workloads.make_workload("cfg2")
plan = engine.plan_from_workload(wl)
xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(5): plan.run(xb, yb)
ts = []
for _ in range(30):
    flush.zero_()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); plan.run(xb, yb); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
ts.sort()
print(f"{os.path.basename(root)} {pkg.__file__[-60:]} median {ts[15]*1e3:.1f} us min {ts[0]*1e3:.1f} us")
