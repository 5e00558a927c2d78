"""Brickify of the cfg2 input alone (NCHW bf16 64x64x56x56 -> 8x8 bricks), L2 flushed before every launch, CUDA
events around each launch; A/B over BDL_BRICKIFY_R (image rows per CTA).    python tools/brickify_probe.py"""
import os, sys, torch
sys.path.insert(0, '.')
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
wl = workloads.make_workload("cfg2")
plan = engine.plan_from_workload(wl)
x = wl["x"].to(device="cuda", dtype=plan.tdtype).contiguous()
xb = plan.alloc_bricked(plan.in_layout)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")   # bench.py's flush: write, then read
MODE = os.environ.get("PROBE_FLUSH", "bench")
def do_flush(it):
    flush.fill_(it & 0xFF)
    if MODE == "bench": flush_rd.sum()
ref = None
for R in sys.argv[1:] or ["1", "2", "4", "8", "2"]:
    os.environ["BDL_BRICKIFY_R"] = R
    ts = []
    for it in range(30):
        do_flush(it)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); plan.brickify(x, out=xb); b.record(); b.synchronize()
        if it >= 5: ts.append(a.elapsed_time(b) * 1e3)
    ts.sort()
    ok = True
    if ref is None: ref = xb.clone()
    else: ok = torch.equal(ref, xb)
    print(f"R={R} median {ts[len(ts)//2]:.2f} us  min {ts[0]:.2f} us  bit-equal {ok}", flush=True)

# floor: a plain device copy of the same bytes (torch copy kernel), same flush and events
dst = torch.empty_like(x)
ts = []
for it in range(30):
    do_flush(it)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); dst.copy_(x); b.record(); b.synchronize()
    if it >= 5: ts.append(a.elapsed_time(b) * 1e3)
ts.sort()
print(f"torch copy of the same {x.numel() * 2 / 1e6:.1f} MB: median {ts[len(ts)//2]:.2f} us  min {ts[0]:.2f} us")
