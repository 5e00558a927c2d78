"""Stress run of the memoized kernels (hang / race hunt): many back-to-back launches of the cfg2 pair kernel under
the wavefront order and several random schedule orders, and of a reduced ResNet-50 on the generic kernel, every
output compared bit for bit with the first.    python tools/stress.py [iterations]"""
import sys, time, torch
sys.path.insert(0, '.')
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
iters = int(sys.argv[1]) if len(sys.argv) > 1 else 2000
t0 = time.time()
for cfg, kw, seeds in (("cfg2", {}, (0, 1, 2, 3)), ("cfg4", dict(N=4, H=112, W=112), (0, 5))):
    wl = workloads.make_workload(cfg, **kw)
    ref = None
    for seed in seeds:
        plan = engine.plan_from_workload(wl, schedule_seed=seed)
        xb = plan.brickify(wl["x"])
        yb = plan.alloc_bricked(plan.out_layout)
        plan.run(xb, yb)
        torch.cuda.synchronize()
        if ref is None:
            ref = yb.clone()
        bad = 0
        n = iters if cfg == "cfg2" else iters // 10
        for i in range(n):
            plan.run(xb, yb)
            if i % 50 == 49:
                torch.cuda.synchronize()
                bad += int(not torch.equal(yb, ref))
        torch.cuda.synchronize()
        bad += int(not torch.equal(yb, ref))
        print(f"{cfg} seed {seed}: {n} runs, {bad} mismatching checks, {time.time() - t0:.1f} s", flush=True)
        assert bad == 0
print("stress ok")
