"""Per-task timeline of the warp-specialized tcgen05 memo kernel (debug).
BDL_TRACE=<cap> python tools/trace_ws.py [mode]   -> gpurun_out/trace_ws_<mode>.json + summary"""
import ctypes, os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("BDL_TRACE", "4096")
import numpy as np, torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads, lib
mode = sys.argv[1] if len(sys.argv) > 1 else "memoized"
wl = workloads.make_workload("cfg2")
plan = engine.plan_from_workload(wl)
plan.set_mode(mode)
xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
for _ in range(3): plan.run(xb, yb)
torch.cuda.synchronize()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); flush.zero_()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(); plan.run(xb, yb); e1.record(); torch.cuda.synchronize()
print("kernel ms (traced run)", e0.elapsed_time(e1), "counters", plan.counters(0))
cap = int(os.environ["BDL_TRACE"])
buf = (ctypes.c_ulonglong * (cap * 8))()
f = lib().bdl_debug_ws_trace; f.restype = ctypes.c_int
n = f(buf, cap)
a = np.frombuffer(buf, dtype=np.uint64).reshape(cap, 8).astype(np.int64)[:n]
a = a[a[:, 7] > 0]
t0 = a[:, 2].min()
rec = []
for r in a:
    rec.append(dict(sm=int(r[0] >> 40), cta=int((r[0] >> 8) & 0xffffffff), l=int(r[0] & 0xff), tile=int(r[1]),
                    q=int(r[2] - t0), dep=int(r[3] - t0) if r[3] else None, loaded=int(r[4] - t0), mma=int(r[5] - t0),
                    acc=int(r[6] - t0), end=int(r[7] - t0)))
print("tasks", len(rec), "span_us", (a[:, 7].max() - t0) / 1e3)
def st(name, v):
    v = np.array(v) / 1e3
    print(f"{name:12s} mean {v.mean():7.2f} p50 {np.median(v):7.2f} p90 {np.percentile(v, 90):7.2f} max {v.max():7.2f} us")
st("dep_wait", [r["dep"] - r["q"] for r in rec if r["dep"] is not None])
st("load", [r["loaded"] - (r["dep"] or r["q"]) for r in rec])
st("load->mma", [r["mma"] - r["loaded"] for r in rec])
st("mma", [r["acc"] - r["mma"] for r in rec])
st("epilogue", [r["end"] - r["acc"] for r in rec])
st("q->end", [r["end"] - r["q"] for r in rec])
# per-CTA busy: first q to last end
by = {}
for r in rec: by.setdefault(r["cta"], []).append(r)
spans = [max(x["end"] for x in v) - min(x["q"] for x in v) for v in by.values()]
st("cta_span", spans)
print("tasks per cta: min", min(len(v) for v in by.values()), "max", max(len(v) for v in by.values()))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(rec, open(f"gpurun_out/trace_ws_{mode}.json", "w"))
