"""Time the cfg2 memo kernel under debug knobs (BDL_WS_DBG bits) to attribute shared-memory traffic."""
import os, sys, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if len(sys.argv) > 1 and sys.argv[1] == "x":
    import torch
    from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
    wl = workloads.make_workload("cfg2", N=int(os.environ.get("NIMG", "64")))
    plan = engine.plan_from_workload(wl)
    plan.set_mode(os.environ.get("MODE", "memoized"))
    xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(5): plan.run(xb, yb)
    ts = []
    for _ in range(20):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); plan.run(xb, yb); b.record(); b.synchronize(); ts.append(a.elapsed_time(b))
    ts.sort()
    print(f"N={wl['N']} mode={os.environ.get('MODE', 'memoized')} dbg={os.environ.get('BDL_WS_DBG','0'):>3s} lag={os.environ.get('BDL_LAG','-')} median {ts[10]*1e3:7.1f} us  min {ts[0]*1e3:7.1f} us")
else:
    for d in (sys.argv[1:] or ["0"]):
        subprocess.run(["timeout", "60", sys.executable, __file__, "x"], env=dict(os.environ, BDL_WS_DBG=d))
