"""Per-task timeline of the warp-specialized tcgen05 memo kernel (debug).
BDL_TRACE=<cap> python tools/trace_ws.py [mode]   -> gpurun_out/trace_ws_<mode>.json + summary
Fields per task (ns): q (loader got it), dep (deps satisfied), loaded (TMA issued), mma0/mma1 (MMA
issue start/end), epi0/epi1 (epilogue start after acc_full / end), sync (store warp got it),
read (staging read out), end (published)."""
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
buf = (ctypes.c_ulonglong * (cap * 16))()
f = lib().bdl_debug_ws_trace; f.restype = ctypes.c_int
n = f(buf, cap)
a = np.frombuffer(buf, dtype=np.uint64).reshape(cap, 16).astype(np.int64)[:n]
a = a[a[:, 11] > 0]
ctarec = a[(a[:, 0] & 0xff) == 255]
a = a[(a[:, 0] & 0xff) != 255]
t0 = a[:, 2].min()
if len(ctarec):
    print("CTA entry (us rel. first task q): min %.2f max %.2f; CTA exit: min %.2f max %.2f" % (
        (ctarec[:, 2].min() - t0) / 1e3, (ctarec[:, 2].max() - t0) / 1e3, (ctarec[:, 11].min() - t0) / 1e3,
        (ctarec[:, 11].max() - t0) / 1e3))
    print("CTA init done (rel. entry) mean %.2f, PDL wait done mean %.2f us" % (
        ((ctarec[:, 3] - ctarec[:, 2]) / 1e3).mean(), ((ctarec[:, 4] - ctarec[:, 2]) / 1e3).mean()))
names = ["q", "dep", "loaded", "mma0", "mma1", "epi0", "epi1", "sync", "read", "end", "emit", "tk", "claimed", "scanned"]
rec = []
for r in a:
    d = dict(sm=int(r[0] >> 40), cta=int((r[0] >> 8) & 0xffffffff), l=int(r[0] & 0xff), tile=int(r[1]))
    for i, nm in enumerate(names):
        d[nm] = int(r[2 + i] - t0) if r[2 + i] else None
    rec.append(d)
print("tasks", len(rec), "span_us", (a[:, 11].max() - t0) / 1e3)
def st(name, v):
    v = np.array([x for x in v if x is not None]) / 1e3
    if len(v): print(f"{name:14s} mean {v.mean():7.2f} p50 {np.median(v):7.2f} p90 {np.percentile(v, 90):7.2f} max {v.max():7.2f} us")
def dif(a_, b_): return [r[b_] - r[a_] for r in rec if r[a_] is not None and r[b_] is not None]
if os.environ.get("BY_LAYER"):
    allrec = rec
    for L_ in sorted({r["l"] for r in allrec}):
        rec = [r for r in allrec if r["l"] == L_]
        print("-- layer", L_)
        for a_, b_ in [("mma1", "epi0"), ("epi0", "epi1"), ("epi1", "sync"), ("sync", "read")]:
            st(f"{a_}->{b_}", dif(a_, b_))
    rec = allrec
PAIR = any(r["emit"] is not None for r in rec)
if PAIR:   # CTA-pair kernel: sync = loader's proxy fence done, read = MMA warp saw both bands (leader records only)
    pairs = [("tk", "claimed"), ("claimed", "scanned"), ("scanned", "emit"), ("emit", "q"), ("q", "dep"), ("dep", "sync"), ("sync", "loaded"), ("loaded", "read"), ("read", "mma0"), ("mma0", "mma1"),
             ("mma1", "epi0"), ("epi0", "epi1"), ("epi1", "end"), ("q", "end")]
else:
    pairs = [("q", "dep"), ("dep", "loaded"), ("loaded", "mma0"), ("mma0", "mma1"), ("mma1", "epi0"),
             ("epi0", "epi1"), ("epi1", "sync"), ("sync", "read"), ("read", "end"), ("q", "end")]
for a_, b_ in pairs:
    st(f"{a_}->{b_}", dif(a_, b_))
by = {}
for r in rec:
    if r["mma0"] is not None: by.setdefault(r["cta"], []).append(r)
gaps, gaps_in = [], []
for v in by.values():
    v.sort(key=lambda r: r["mma0"])
    for x, y in zip(v, v[1:]): gaps.append(y["mma0"] - x["mma1"])
    if PAIR:
        for x, y in zip(v, v[1:]):
            if y["read"] is not None: gaps_in.append(max(0, y["read"] - x["mma1"]))
st("mma idle gap", gaps)
if PAIR:
    em = []
    for v in by.values():
        e = sorted(x["emit"] for x in v if x["emit"] is not None)
        em += [b - a for a, b in zip(e, e[1:])]
    st("emit interval", em)
if PAIR: st("mma waits bands", gaps_in)
spans = [max(x["end"] for x in v) - min(x["q"] for x in v) for v in by.values()]
starts = [min(x["mma0"] for x in v) for v in by.values()]
ends = [max(x["mma1"] for x in v) for v in by.values()]
busy = [sum(x["mma1"] - x["mma0"] for x in v) for v in by.values()]
st("first mma0", starts); st("last mma1", ends); st("mma busy/cta", busy)
st("cta_span", spans)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(rec, open(f"gpurun_out/trace_ws_{mode}.json", "w"))
