"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Tolerances (BASELINE.json north_star):
  * layout / indexing: bit-exact;
  * fp32 CUDA-core path: max|y - ref| / max|ref| <= 1e-5 against the fp64 oracle with fp32 storage;
  * bf16 tcgen05 / bf16 storage paths: <= 2e-2 against the oracle emulating bf16 storage rounding.
Modes (padded / memoized / unmerged) use one accumulation order per element, so they must agree
bit for bit with each other.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads

pytestmark = pytest.mark.gpu

TOL = {"f32": 1e-5, "bf16": 2e-2}


def rel_err(y, ref):
    y = np.asarray(y, dtype=np.float64)
    return float(np.max(np.abs(y - ref)) / max(np.max(np.abs(ref)), 1e-30))


def oracle_out(wl, images=None):
    x = wl["x"].numpy()
    if images is not None:
        x = x[images]
    return oracle.run_graph(wl["layers"], x, wl["weights"], wl["biases"], dtype=wl["dtype"])


# ---------------------------------------------------------------- layout (bit-exact)
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("shape,brick", [
    ((1, 8, 1, 32, 32), (1, 1, 8, 8)),
    ((3, 5, 1, 20, 13), (1, 1, 8, 8)),
    ((2, 64, 1, 56, 56), (1, 1, 8, 8)),
    ((3, 3, 1, 17, 30), (2, 1, 4, 16)),
    ((1, 32, 9, 10, 7), (1, 4, 4, 4)),
])
def test_brickify_bitexact(dtype, shape, brick):
    N, C, D, H, W = shape
    nsp = 3 if D > 1 or brick[1] > 1 else 2
    tdt = torch.float32 if dtype == "f32" else torch.bfloat16
    x = torch.randn(shape, generator=torch.Generator().manual_seed(7)).to(tdt)
    lo = engine.make_layout(nsp, N, C, D, H, W, brick, 0 if dtype == "f32" else 1)
    dst = torch.empty(int(lo.total_bytes), dtype=torch.uint8, device="cuda")
    import ctypes
    from paper_conf_icpp_lakshminarasimhan24_b200 import check, lib
    xd = x.cuda().contiguous()
    check(lib().bdl_brickify(ctypes.byref(lo), ctypes.c_void_p(xd.data_ptr()), ctypes.c_void_p(dst.data_ptr()), None))
    got = dst.view(tdt).float().cpu().numpy().astype(np.float64)
    ref = oracle.brickify(x.float().numpy(), brick, lo.c_pad)
    np.testing.assert_array_equal(got, ref)
    back = torch.empty(shape, dtype=tdt, device="cuda")
    check(lib().bdl_unbrickify(ctypes.byref(lo), ctypes.c_void_p(dst.data_ptr()), ctypes.c_void_p(back.data_ptr()), None))
    assert torch.equal(back.cpu(), x)


def test_brickify_with_brickmap():
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "fig6_brickinfo.json")))
    bm = np.array(g["brickmap"], dtype=np.int32).reshape(-1)
    x = torch.randn(1, 8, 1, 16, 16, generator=torch.Generator().manual_seed(3))
    wl = dict(layers=workloads.make_layers("cfg1", C=8, nlayers=1))
    w = [torch.randn(8, 8, 1, 3, 3, generator=torch.Generator().manual_seed(4)) * 0.2]
    b = [torch.zeros(8)]
    plan = engine.Plan(wl["layers"], w, b, 1, 8, 1, 16, 16, 2, "f32", (1, 1, 4, 4), brickmap=bm)
    xb = plan.brickify(x)
    ref = oracle.brickify(x.numpy(), (1, 1, 4, 4), 8, brickmap=bm)
    np.testing.assert_array_equal(xb.view(torch.float32).cpu().numpy().astype(np.float64), ref)
    y = plan.unbrickify(plan.run(xb)).cpu().numpy()
    yref = oracle.run_graph(wl["layers"], x.numpy(), w, b, dtype="f32")
    assert rel_err(y, yref) <= 1e-5


# ---------------------------------------------------------------- cfg1: fp32 CUDA-core chain
@pytest.mark.parametrize("size", [dict(), dict(N=3, H=27, W=41), dict(N=2, C=5, H=16, W=8)])
def test_cfg1_modes_vs_oracle(size):
    wl = workloads.make_workload("cfg1", **size)
    ref = oracle_out(wl)
    plan = engine.plan_from_workload(wl)
    outs = {}
    for mode in ("padded", "memoized", "unmerged"):
        plan.set_mode(mode)
        outs[mode] = plan.forward(wl["x"]).cpu().numpy()
        assert rel_err(outs[mode], ref) <= TOL["f32"], mode
    np.testing.assert_array_equal(outs["padded"], outs["memoized"])
    np.testing.assert_array_equal(outs["padded"], outs["unmerged"])


def test_cfg1_memo_counters_exactly_once():
    wl = workloads.make_workload("cfg1", N=2, H=40, W=40, nlayers=4)
    plan = engine.plan_from_workload(wl)
    plan.set_mode("memoized")
    plan.forward(wl["x"])
    c = plan.counters(0)
    nb = 2 * 5 * 5
    # M1: every (layer, brick) computed exactly once; M2: successful claims == bricks (2 compulsory
    # atomics per brick: the claim and the release)
    assert c["computed"] == 4 * nb
    assert c["cas_ok"] == 4 * nb


# ---------------------------------------------------------------- cfg2: bf16 tcgen05 band kernel
@pytest.mark.parametrize("size", [
    dict(N=2, H=20, W=20),            # ragged vs 8x8 bricks
    dict(N=1, H=56, W=56),            # full image shape
    dict(N=3, C=32, H=16, W=24),
    dict(N=2, C=16, H=9, W=33),
    dict(N=1, C=128, H=24, W=24),
])
def test_cfg2_tc_modes_vs_oracle(size):
    wl = workloads.make_workload("cfg2", **size)
    ref = oracle_out(wl)
    plan = engine.plan_from_workload(wl)
    # C <= 64: the band kernels; C = 128 chains run on the generic kernel (the warp-specialized band kernel's
    # weights-resident design holds C <= 64)
    assert plan.subgraphs()[0]["kernel"] == ("tcgen05 band" if wl["C"] <= 64 else "tcgen05 generic")
    outs = {}
    for mode in ("padded", "memoized", "unmerged"):
        plan.set_mode(mode)
        outs[mode] = plan.forward(wl["x"]).float().cpu().numpy()
        assert rel_err(outs[mode], ref) <= TOL["bf16"], (mode, rel_err(outs[mode], ref))
    np.testing.assert_array_equal(outs["padded"], outs["memoized"])
    np.testing.assert_array_equal(outs["memoized"], outs["unmerged"])


def test_cfg2_tc_memo_counters():
    wl = workloads.make_workload("cfg2", N=4, H=40, W=40)
    plan = engine.plan_from_workload(wl)
    plan.set_mode("memoized")
    plan.forward(wl["x"])
    c = plan.counters(0)
    tb = plan.subgraphs()[0]["tc_band"]
    tasks = 2 * 4 * -(-40 // tb)   # layers x images x Tb-row bands (full-width tiles)
    assert c["computed"] == tasks and c["cas_ok"] == tasks


def test_cfg2_full_size_sampled():
    """BASELINE configs[1] at full size (N=64, 56x56, C=64), the bench's launch configuration;
    images 0 and 63 checked against the oracle element by element."""
    wl = workloads.make_workload("cfg2")
    plan = engine.plan_from_workload(wl)
    sg = plan.subgraphs()[0]
    assert sg["kernel"] == "tcgen05 band" and sg["mode"] == "memoized"
    y = plan.forward(wl["x"]).float().cpu().numpy()
    ref = oracle_out(wl, images=[0, 63])
    assert rel_err(y[[0, 63]], ref) <= TOL["bf16"]
    plan.set_mode("padded")
    y2 = plan.forward(wl["x"]).float().cpu().numpy()
    np.testing.assert_array_equal(y, y2)


def test_repeat_runs_epoch_tags():
    """Memo tags are epoch-stamped: back-to-back runs without re-prepare stay correct."""
    wl = workloads.make_workload("cfg2", N=2, H=16, W=16)
    plan = engine.plan_from_workload(wl)
    plan.set_mode("memoized")
    xb = plan.brickify(wl["x"])
    first = plan.unbrickify(plan.run(xb)).cpu()
    for _ in range(5):
        again = plan.unbrickify(plan.run(xb)).cpu()
        assert torch.equal(first, again)


# ---------------------------------------------------------------- other configs (small shapes)
def test_cfg5_3d_small():
    wl = workloads.make_workload("cfg5", D=12, H=12, W=12, C=8)
    ref = oracle_out(wl)
    plan = engine.plan_from_workload(wl)
    for mode in ("padded", "memoized", "unmerged"):
        plan.set_mode(mode)
        y = plan.forward(wl["x"]).float().cpu().numpy()
        assert rel_err(y, ref) <= TOL["bf16"], mode


def test_cfg3_vgg_small():
    wl = workloads.make_workload("cfg3", N=1, H=32, W=32)
    ref = oracle_out(wl)
    plan = engine.plan_from_workload(wl)
    y = plan.forward(wl["x"]).float().cpu().numpy()
    assert rel_err(y, ref) <= TOL["bf16"]


def test_cfg4_resnet50_small():
    wl = workloads.make_workload("cfg4", N=1, H=64, W=64)
    ref = oracle_out(wl)
    plan = engine.plan_from_workload(wl)
    y = plan.forward(wl["x"]).float().cpu().numpy()
    assert rel_err(y, ref) <= TOL["bf16"]


# ---------------------------------------------------------------- schedule invariance
def test_memo_schedule_invariance():
    """Any task order gives bit-identical results and exactly-once execution: the scheduler claims
    not-started dependencies first (Fig 2d recursion) and waits for in-progress ones."""
    wl = workloads.make_workload("cfg2", N=3, H=24, W=24)
    ref = None
    for seed in (0, 1, 7, 123):
        plan = engine.plan_from_workload(wl, schedule_seed=seed)
        plan.set_mode("memoized")
        y = plan.forward(wl["x"]).float().cpu().numpy()
        c = plan.counters(0)
        tb = plan.subgraphs()[0]["tc_band"]
        tasks = 2 * 3 * -(-24 // tb)
        assert c["computed"] == tasks and c["cas_ok"] == tasks, (seed, c)
        if ref is None:
            ref = y
            assert rel_err(y, oracle_out(wl)) <= TOL["bf16"]
        else:
            np.testing.assert_array_equal(y, ref)


# ---------------------------------------------------------------- full-size configurations, sampled
def test_cfg5_full_size_sampled_crops():
    """cfg5 at full size (1 x 32 x 128^3, four 3x3x3 layers, 4^3 bricks); the oracle evaluates crops
    whose interior (4 voxels from any crop face that is not a volume face) equals the full result."""
    wl = workloads.make_workload("cfg5")
    plan = engine.plan_from_workload(wl)
    y = plan.forward(wl["x"]).float().cpu().numpy()
    x = wl["x"].numpy()
    for lo, hi in [((0, 0, 0), (20, 20, 20)), ((60, 100, 30), (84, 128, 54))]:
        sl = tuple(slice(a, b) for a, b in zip(lo, hi))
        crop = x[(slice(None), slice(None)) + sl]
        ref = oracle.run_graph(wl["layers"], crop, wl["weights"], wl["biases"], dtype="bf16")
        keep = tuple(slice(0 if a == 0 else 4, (b - a) if b == 128 else (b - a) - 4) for a, b in zip(lo, hi))
        got = y[(slice(None), slice(None)) + sl][(slice(None), slice(None)) + keep]
        assert rel_err(got, ref[(slice(None), slice(None)) + keep]) <= TOL["bf16"]


@pytest.mark.parametrize("cfg", ["cfg3", "cfg4"])
def test_full_resolution_single_image(cfg):
    """VGG-16 / ResNet-50 backbone at the paper's 224x224 resolution (one image), whole graph
    partitioned by the planner, against the oracle."""
    wl = workloads.make_workload(cfg, N=1)
    ref = oracle_out(wl)
    plan = engine.plan_from_workload(wl)
    y = plan.forward(wl["x"]).float().cpu().numpy()
    assert rel_err(y, ref) <= TOL["bf16"]


@pytest.mark.parametrize("cfg", ["cfg3", "cfg4"])
def test_full_batch_sampled(cfg):
    """VGG-16 at N=128 / ResNet-50 at N=256: the bench's batch sizes and launch configuration (several
    image groups in the generic kernel's task order, padded CTA blocks grown to whole-image bands).
    Images 0 and N-1 are checked against the oracle element by element, and bit for bit against a
    one-image plan of the same graph (merged execution only reorders work, L363-365; one K-order
    per element in every geometry and mode)."""
    wl = workloads.make_workload(cfg)
    N = wl["N"]
    plan = engine.plan_from_workload(wl)
    y = plan.forward(wl["x"]).float().cpu().numpy()
    del plan
    torch.cuda.empty_cache()
    ref = oracle_out(wl, images=[0, N - 1])
    assert rel_err(y[[0, N - 1]], ref) <= TOL["bf16"], rel_err(y[[0, N - 1]], ref)
    one = workloads.make_workload(cfg, N=1)
    p1 = engine.plan_from_workload(one)
    for n in (0, N - 1):
        y1 = p1.forward(wl["x"][n:n + 1]).float().cpu().numpy()
        np.testing.assert_array_equal(y[n:n + 1], y1)


@pytest.mark.parametrize("case", ["cfg2_memo", "cfg2_unmerged", "cfg2_padded", "cfg2_c32", "cfg4_small", "cfg1_f32"])
def test_run_dense_equals_run_then_unbrickify(case):
    """bdl_run_dense (unbrickify fused into the last subgraph's epilogue where its kernel supports it, else staged +
    one unbrickify launch) gives exactly the bytes of bdl_run + bdl_unbrickify (the layout conversion is exact,
    L742-743), and repeated runs stay equal (run state on the device)."""
    if case.startswith("cfg2"):
        kw = dict(N=3, H=24, W=40) if case != "cfg2_c32" else dict(N=2, C=32, H=20, W=24)
        wl = workloads.make_workload("cfg2", **kw)
        mode = {"cfg2_memo": "memoized", "cfg2_unmerged": "unmerged", "cfg2_padded": "padded"}.get(case, "memoized")
    elif case == "cfg4_small":
        wl, mode = workloads.make_workload("cfg4", N=2, H=64, W=64), None
    else:
        wl, mode = workloads.make_workload("cfg1", N=2, H=24, W=16), "memoized"
    plan = engine.plan_from_workload(wl)
    if mode:
        plan.set_mode(mode)
    xb = plan.brickify(wl["x"])
    ref = plan.unbrickify(plan.run(xb))
    for _ in range(3):
        got = plan.run_dense(xb)
        assert torch.equal(got, ref), case
    assert rel_err(got.float().cpu().numpy(), oracle_out(wl)) <= TOL[wl["dtype"]]
