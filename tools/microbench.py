"""B200 re-run of the paper's memo-overhead microbenchmarks (§4.4).

  * T_atomic: the latency of the memo table's atomics (paper: 87.45 ns per CAS on A100, SURVEY Q4 reading):
    dependent atomicCAS chains on a status word, uncontended (own word per CTA), contended (one word for all
    CTAs), and the whole compulsory protocol of one memo unit (ld.acquire + CAS 0 -> 1 + st.release 2).
  * T_brick: the compute time of one memo unit of the paper's microbenchmark layer (3x3x3 conv, 64 -> 64 channels,
    valid padding; paper: 6.72 us per brick with cuDNN on A100): our unit is a generic-kernel task
    (an output tile of one depth plane); reported as the amortized time per task per SM of a full layer launch and
    as the launch time of a single-task volume.
  * The ratio T_atomic x 2 / T_unit is the compulsory-atomics overhead fraction per unit (paper: Fig 8).
    python tools/microbench.py [--out profiles/r02_microbench.txt]
"""
import argparse
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_icpp_lakshminarasimhan24_b200 import build, engine, workloads as W  # noqa: E402


def cas(lib, ctas, mode, iters=20000):
    ns, ff = ctypes.c_double(), ctypes.c_double()
    rc = lib.bdl_mb_cas(ctas, iters, mode, ctypes.byref(ns), ctypes.byref(ff))
    assert rc == 0, rc
    return ns.value, ff.value


def layer_time(D, reps=5):
    """One 3x3x3 64->64 valid layer over a D^3 volume (bricks 4^3): ms per launch and tasks (memo units)."""
    layers = [W.conv(64, 64, 3, 1, 0, nsp=3)]
    wl = W.make_graph_workload(layers, 1, 64, D, D, D, 3, (1, 4, 4, 4), "bf16", seed=5)
    plan = engine.plan_from_workload(wl)
    xb = plan.brickify(wl["x"])
    yb = plan.alloc_bricked(plan.out_layout)
    for _ in range(3):
        plan.run(xb, yb)
    torch.cuda.synchronize()
    plan.prepare()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in ev:
        a.record()
        plan.run(xb, yb)
        b.record()
    torch.cuda.synchronize()
    ms = sorted(a.elapsed_time(b) for a, b in ev)[reps // 2]
    tasks = plan.counters(0)["computed"] // reps
    return ms, tasks


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    lib = ctypes.CDLL(build.build_microbench())
    lib.bdl_mb_cas.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                               ctypes.POINTER(ctypes.c_double)]
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    lines = [f"# B200 memo microbenchmarks ({torch.cuda.get_device_name(0)}, {nsm} SMs) -- tools/microbench.py",
             "# T_atomic (paper A100: 87.45 ns per CAS, L1082-1104)"]
    res = {}
    for ctas in (1, nsm):
        for mode, name in ((0, "CAS uncontended (own word)"), (1, "CAS contended (one word)"),
                           (2, "claim+publish (ld.acquire, CAS 0->1, st.release 2)")):
            ns, ff = cas(lib, ctas, mode)
            res[(ctas, mode)] = ns
            lines.append(f"  {ctas:4d} CTAs  {name:52s} {ns:8.1f} ns/op   failed CAS {100 * ff:5.1f} %")
    lines.append("# T_brick analogue: 3x3x3 conv 64->64 valid (SURVEY Q2), generic tcgen05 kernel (paper A100: 6.72 us)")
    for D in (12, 112):
        ms, tasks = layer_time(D)
        per_task_sm = ms * 1e3 * min(nsm, tasks) / max(tasks, 1)
        lines.append(f"  volume {D:3d}^3: {tasks:6d} units, {ms * 1e3:9.1f} us per launch, "
                     f"{per_task_sm:7.2f} us per unit per SM (amortized)")
        res[D] = per_task_sm
    t_unit = res[112]
    lines.append(f"# compulsory atomics per unit (claim + publish) / unit compute time: "
                 f"{res[(nsm, 2)] / 1e3 / t_unit * 100:.2f} % (paper A100: 2 x 87.45 ns / 6.72 us = "
                 f"{2 * 87.45 / 6720 * 100:.2f} %)")
    txt = "\n".join(lines)
    print(txt)
    if a.out:
        with open(a.out, "w") as f:
            f.write(txt + "\n")


if __name__ == "__main__":
    main()
