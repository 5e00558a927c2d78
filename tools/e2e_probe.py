"""Where the e2e (host-to-host) number of the cfg2 bench stands against PCIe: pinned H2D / D2H copy times of one step's
input and output (25.7 MB each), both directions concurrently, and the serving pipeline (engine.HostPipeline) at 2-6
buffer slots.    python tools/e2e_probe.py   (on a B200)"""
import sys, torch, time
sys.path.insert(0, '.')
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
wl = workloads.make_workload("cfg2")
plan = engine.plan_from_workload(wl)
x_host = wl["x"].to(plan.tdtype).contiguous().pin_memory()
y_host = torch.empty_like(x_host).pin_memory()
xd = torch.empty_like(x_host, device="cuda"); yd = torch.empty_like(x_host, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def t(fn, n=20):
    torch.cuda.synchronize(); a = time.perf_counter()
    for _ in range(n): fn()
    torch.cuda.synchronize(); return (time.perf_counter() - a) / n * 1e3
print("H2D ms", t(lambda: xd.copy_(x_host, non_blocking=True)))
print("D2H ms", t(lambda: y_host.copy_(yd, non_blocking=True)))
def both():
    with torch.cuda.stream(s1): xd.copy_(x_host, non_blocking=True)
    with torch.cuda.stream(s2): y_host.copy_(yd, non_blocking=True)
print("H2D||D2H ms", t(both))
for slots in (2, 3, 4, 6):
    pipe = engine.HostPipeline(plan, slots=slots)
    pipe.run([x_host] * 4)
    torch.cuda.synchronize()
    K = 40
    a = time.perf_counter(); pipe.run([x_host] * K, on_output=lambda k, y: None); torch.cuda.synchronize()
    ms = (time.perf_counter() - a) / K * 1e3
    print("slots", slots, "ms/step", round(ms, 3), "img/s", round(64 / ms * 1e3))
