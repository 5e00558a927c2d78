"""A/B the full cfg2 step (brickify + merged subgraph + unbrickify, L2 flushed before each step) of another
checkout: python tools/ab_step.py <repo root>"""
import os, sys
root = os.path.abspath(sys.argv[1])
sys.path.insert(0, root)
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
wl = workloads.make_workload(sys.argv[2] if len(sys.argv) > 2 else "cfg2")
plan = engine.plan_from_workload(wl)
x = wl["x"].to("cuda", plan.tdtype).contiguous()
xb = plan.alloc_bricked(plan.in_layout); yb = plan.alloc_bricked(plan.out_layout)
y = torch.empty((plan.out_layout.N, plan.out_layout.C, plan.out_layout.D, plan.out_layout.H, plan.out_layout.W),
                dtype=plan.tdtype, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); rd = torch.ones(64 << 20, device="cuda")
def step():
    plan.brickify(x, out=xb); plan.run(xb, yb); plan.unbrickify(yb, out=y)
for _ in range(5): step()
ts = [[], [], [], []]
for _ in range(20):
    flush.zero_(); rd.sum()
    e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    e[0].record(); plan.brickify(x, out=xb); e[1].record(); plan.run(xb, yb); e[2].record(); plan.unbrickify(yb, out=y); e[3].record()
    e[3].synchronize()
    for i in range(3): ts[i].append(e[i].elapsed_time(e[i + 1]) * 1e3)
    ts[3].append(e[0].elapsed_time(e[3]) * 1e3)
med = [sorted(t)[10] for t in ts]
print(f"{os.path.basename(root):6s} brickify {med[0]:.1f} run {med[1]:.1f} unbrickify {med[2]:.1f} step {med[3]:.1f} us")
