"""The CTA-pair tcgen05 kernel (chain_tc_pair.cu) for C = 64 3x3 chains over full-width bands.

It replaces the single-CTA band kernel (chain_tc_ws.cu) for memoized and unmerged execution when its geometry fits.
Both issue, per output element, the same sequence of K = 16 products (tap-major, 16-channel steps inner), so the pair
kernel must reproduce the single-CTA kernel bit for bit (BDL_NO_PAIR=1 selects the latter, read at plan and launch
time); against the oracle it meets the bf16 tolerance like every tensor-core path.  Cases: the bench shape, a ragged
band count (H = 44: the last band has 2 rows, one M tile), one image (every pair has an idle half: each (step, layer)
run of the pair order is padded), and a 3-layer chain (all layers' weights resident: a shorter band).
"""
import os

import numpy as np
import pytest
import torch

from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
from test_gpu_parity import TOL, oracle_out, rel_err

pytestmark = pytest.mark.gpu


def run_modes(wl, modes=("memoized", "unmerged")):
    plan = engine.plan_from_workload(wl)
    outs = {}
    for m in modes:
        plan.set_mode(m)
        outs[m] = plan.forward(wl["x"]).float().cpu().numpy()
    return plan, outs


def with_env(key, val, fn):
    old = os.environ.get(key)
    os.environ[key] = val
    try:
        return fn()
    finally:
        if old is None:
            del os.environ[key]
        else:
            os.environ[key] = old


@pytest.mark.parametrize("shape", [dict(N=64), dict(N=3, H=44), dict(N=1)])
def test_pair_equals_single_cta_kernel(shape):
    wl = workloads.make_workload("cfg2", **shape)
    plan, pair = run_modes(wl)
    assert plan.subgraphs()[0]["cta_pair"]
    def single_cta():
        plan1, outs = run_modes(wl)
        assert not plan1.subgraphs()[0]["cta_pair"]
        return outs

    single = with_env("BDL_NO_PAIR", "1", single_cta)
    for m in pair:
        np.testing.assert_array_equal(pair[m], single[m])
    np.testing.assert_array_equal(pair["memoized"], pair["unmerged"])
    imgs = [0, wl["N"] - 1] if wl["N"] > 2 else None
    ref = oracle_out(wl, images=imgs) if imgs else oracle_out(wl)
    got = pair["memoized"][imgs] if imgs else pair["memoized"]
    assert rel_err(got, ref) <= TOL["bf16"]


def test_pair_three_layer_chain():
    """conv-ReLU x3 (+ input residual on the last): three layers' weights stay resident, so the band is shorter."""
    C, N, H, W = 64, 4, 56, 56
    layers = [workloads.conv(C, C), workloads.conv(C, C), workloads.conv(C, C, res=-1, wscale=0.5)]
    wl = workloads.make_graph_workload(layers, N, C, 1, H, W, 2, (1, 1, 8, 8), "bf16")
    plan, outs = run_modes(wl, ("memoized", "unmerged", "padded"))
    sg = plan.subgraphs()
    assert len(sg) == 1 and sg[0]["cta_pair"] and sg[0]["tc_band"] < 6
    np.testing.assert_array_equal(outs["memoized"], outs["unmerged"])
    np.testing.assert_array_equal(outs["memoized"], outs["padded"])
    assert rel_err(outs["memoized"], oracle_out(wl)) <= TOL["bf16"]
    plan.set_mode("memoized")   # (re-prepares: counters from zero)
    plan.forward(wl["x"])
    c = plan.counters(0)
    tasks = 3 * N * -(-H // sg[0]["tc_band"])   # every (layer, band) task computed exactly once
    assert c["computed"] == tasks and c["cas_ok"] == tasks, c


@pytest.mark.parametrize("brick,H,W", [((1, 1, 4, 4), 36, 52), ((1, 1, 8, 16), 30, 48), ((1, 1, 2, 8), 17, 40)])
def test_pair_other_bricks(brick, H, W):
    """Other brick shapes: the band row is W + Bw pixels (the out-of-map brick is the zero pad) and TMA boxes never
    cross a brick row, so the pair kernel must match the single-CTA kernel bit for bit and the oracle."""
    layers = workloads.make_layers("cfg2")
    wl = workloads.make_graph_workload(layers, 3, 64, 1, H, W, 2, brick, "bf16", seed=7)
    plan, pair = run_modes(wl)
    assert plan.subgraphs()[0]["cta_pair"]

    def single_cta():
        plan1, outs = run_modes(wl)
        assert not plan1.subgraphs()[0]["cta_pair"]
        return outs

    single = with_env("BDL_NO_PAIR", "1", single_cta)
    for m in pair:
        np.testing.assert_array_equal(pair[m], single[m])
    assert rel_err(pair["memoized"], oracle_out(wl)) <= TOL["bf16"]
