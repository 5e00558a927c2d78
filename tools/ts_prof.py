"""Per-role busy/wait split of the tap-shared memo kernel (debug: BDL_WS_DBG=256 + BDL_TRACE)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["BDL_TRACE"] = "4096"
os.environ["BDL_WS_DBG"] = str(256 | int(os.environ.get("EXTRA_DBG", "0")))
import numpy as np, torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads, lib
mode = sys.argv[1] if len(sys.argv) > 1 else "memoized"
wl = workloads.make_workload("cfg2")
plan = engine.plan_from_workload(wl)
plan.set_mode(mode)
xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
for _ in range(3): plan.run(xb, yb)
torch.cuda.synchronize()
plan.run(xb, yb); torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * (4096 * 12))()
f = lib().bdl_debug_ws_trace; f.restype = ctypes.c_int
f(buf, 4096)
a = np.frombuffer(buf, dtype=np.uint64).astype(np.int64)[:148 * 16].reshape(148, 8, 2)
names = ["sched(q_empty)", "loader(q_full,in_empty,pub_done)", "mma(in_full)", "publisher(desc,stored)", "epi(desc,acc_full)", "mma(acc_empty)", "epi(bar.sync xch)"]
for r, nm in enumerate(names):
    w, t = a[:, r, 0], a[:, r, 1]
    ok = t > 0
    print(f"{nm:36s} wait {w[ok].mean():9.0f} of {t[ok].mean():9.0f} cycles ({100*w[ok].mean()/max(1,t[ok].mean()):5.1f}% waiting)")
