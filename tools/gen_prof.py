"""Per-role wait/busy split of the generic tcgen05 kernel, per subgraph (debug, BDL_GEN_PROF).
    python tools/gen_prof.py cfg4 [subgraph ...]"""
import ctypes, os, sys
sys.path.insert(0, os.environ.get("BDL_ROOT") or os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["BDL_GEN_PROF"] = "1"
import numpy as np, torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads, lib
cfg = sys.argv[1]
wl = workloads.make_workload(cfg)
ml = int(os.environ.get("MAXL", "0"))
plan = engine.plan_from_workload(wl, max_subgraph_layers=ml) if ml else engine.plan_from_workload(wl)
xb = plan.brickify(wl["x"]); yb = plan.alloc_bricked(plan.out_layout)
plan.run(xb, yb); torch.cuda.synchronize()
sgs = plan.subgraphs()
ids = [int(a) for a in sys.argv[2:]] or range(len(sgs))
f = lib().bdl_debug_gen_prof; f.restype = ctypes.c_int
names = ["ld q_full", "ld deps", "ld in_empty", "ld total", "wp wempty", "wp total", "mma desc", "mma acc_empty",
         "mma in_full", "mma wfull", "mma total", "epi desc", "epi acc_full", "epi bar", "epi total", "mma fence"]
for i in ids:
    if sgs[i]["kernel"] != "tcgen05 generic":
        continue
    plan.run_subgraph(i, xb, yb); torch.cuda.synchronize()
    buf = (ctypes.c_ulonglong * (1024 * 32))()
    f(buf, 1024)
    a = np.frombuffer(buf, dtype=np.uint64).reshape(1024, 32).astype(np.float64)
    a = a[a[:, 3] > 0]
    m = a.mean(axis=0)
    ls = wl["layers"][sgs[i]["first"]:sgs[i]["last"] + 1]
    desc = " ".join(f"{l['kind'][0]}{l['cin']}>{l['cout']}k{l['k'][-1]}s{l['stride'][-1]}" for l in ls)
    print(f"sg {i} {sgs[i]['mode']} {desc}: ctas {len(a)}  total {m[14]/1.9e3:.0f} us")
    print("   " + "  ".join(f"{n} {100*m[k]/max(m[14],1):.0f}%" for k, n in enumerate(names) if k not in (3, 5, 10, 14)))
    print(f"   per-role totals (us): loader {m[3]/1.9e3:.0f} wprod {m[5]/1.9e3:.0f} mma {m[10]/1.9e3:.0f} epi {m[14]/1.9e3:.0f}")
    nt = max(m[19], 1)
    print(f"   per task (us, {nt:.0f} tasks/CTA): epi items {m[17]/nt/1.9e3:.2f} (tmem {m[16]/nt/1.9e3:.2f}) "
          f"publish {m[18]/nt/1.9e3:.2f} bar {m[13]/nt/1.9e3:.2f} acc_wait {m[12]/nt/1.9e3:.2f} | "
          f"loader issue {m[20]/nt/1.9e3:.2f} bar1 {m[21]/nt/1.9e3:.2f} deps {m[1]/nt/1.9e3:.2f} in_empty {m[2]/nt/1.9e3:.2f}")
