"""Per-task timeline of the tcgen05 memo kernel (debug): BDL_TRACE=<cap> python tools/trace_tc.py"""
import ctypes, os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("BDL_TRACE", "4096")
import numpy as np, torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads, lib
wl = workloads.make_workload("cfg2")
plan = engine.plan_from_workload(wl)
mode = sys.argv[1] if len(sys.argv) > 1 else "memoized"
plan.set_mode(mode)
xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
for _ in range(3): plan.run(xb, yb)
plan.prepare()           # zero counters (trace index)
torch.cuda.synchronize()
plan.run(xb, yb); torch.cuda.synchronize()
cap = int(os.environ["BDL_TRACE"])
buf = (ctypes.c_ulonglong * (cap * 7))()
lib().bdl_debug_trace_copy(buf, cap)
a = np.frombuffer(buf, dtype=np.uint64).reshape(cap, 7).astype(np.int64)
a = a[a[:, 2] > 0]
t0 = a[:, 2].min()
rec = []
for r in a:
    rec.append(dict(sm=int(r[0] >> 32), cta=int((r[0] >> 8) & 0xffffff), l=int(r[0] & 0xff), tile=int(r[1]),
                    ctrl=int(r[3]-r[2]), load=int(r[4]-r[3]), mma=int(r[5]-r[4]), epi=int(r[6]-r[5]),
                    start=int(r[2]-t0), end=int(r[6]-t0)))
print("tasks", len(rec), "span_us", (a[:, 6].max() - t0) / 1e3)
for k in ("ctrl", "load", "mma", "epi"):
    v = np.array([x[k] for x in rec]); print(k, "mean_us %.2f p50 %.2f max %.2f" % (v.mean()/1e3, np.median(v)/1e3, v.max()/1e3))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(rec, open(f"gpurun_out/trace_{mode}.json", "w"))
