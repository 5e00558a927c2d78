import os, sys
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
wl = workloads.make_workload("cfg2")
plan = engine.plan_from_workload(wl)
x = wl["x"].to("cuda", plan.tdtype).contiguous()
xb = plan.alloc_bricked(plan.in_layout); yb = plan.alloc_bricked(plan.out_layout)
y = torch.empty((64, 64, 1, 56, 56), dtype=plan.tdtype, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); rd = torch.ones(64 << 20, device="cuda")
for _ in range(5): plan.unbrickify(plan.run(plan.brickify(x, out=xb), yb), out=y)
for inner in (True, False, True, False):
    ts = []
    for _ in range(20):
        flush.zero_(); rd.sum()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        e[0].record(); plan.brickify(x, out=xb)
        if inner: e[1].record()
        plan.run(xb, yb)
        if inner: e[2].record()
        plan.unbrickify(yb, out=y); e[3].record(); e[3].synchronize()
        ts.append(e[0].elapsed_time(e[3]) * 1e3)
    print("inner events" if inner else "outer only  ", "step median %.1f us" % sorted(ts)[10])
