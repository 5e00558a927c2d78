"""Memo-table atomics breakdown on B200 (Fig 8 / §4.4).

For each memoized subgraph: units computed, successful CAS claims (compulsory: one claim + one release
store per unit, L1147-1149), failed claims (conflicts: the unit was already claimed by another worker),
and dependency polls, under the locality-aware wavefront order and under a seeded random order
(schedule_seed), which is what the paper's arbitrary thread-block order corresponds to.
    python tools/memo_breakdown.py [cfg ...]
"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads


def run(cfg, seed):
    wl = workloads.make_workload(cfg)
    plan = engine.plan_from_workload(wl, **({"schedule_seed": seed} if seed else {}))
    plan.set_mode("memoized")
    xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
    plan.run(xb, yb); torch.cuda.synchronize()
    for i, s in enumerate(plan.subgraphs()):
        if s["last"] == s["first"]:
            continue
        plan.prepare()                       # zero the counters
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); plan.run_subgraph(i, xb, yb); b.record(); b.synchronize()
        c = plan.counters(i)
        print(f"{cfg} sg{i} [{s['first']},{s['last']}] {s['kernel']:16s} order={'random' if seed else 'wavefront'}: "
              f"{a.elapsed_time(b):7.3f} ms  units {c['computed']}  claims {c['cas_ok']}  "
              f"compulsory atomics {2 * c['computed']}  conflicts {c['cas_fail']}  polls {c['spins']}")
        if i > 3:
            break


for cfg in (sys.argv[1:] or ["cfg1", "cfg2", "cfg5"]):
    for seed in (0, 1234):
        run(cfg, seed)
