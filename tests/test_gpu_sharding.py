"""Spatial D-slab sharding of cfg5 volumes on the GPU: every rank's plan runs on its slab
extended by one brick plane of halo per face; the ranks are emulated in one process on one GPU (the halo
exchange is the same byte ranges as the torch.distributed path, tests/test_sharding.py checks those over
gloo).  Stitched output == unsharded output bit for bit (same kernels, same per-voxel K order), and within
the bf16 tolerance of the oracle."""
import os
import sys

import numpy as np
import pytest
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, parallel, workloads  # noqa: E402

pytestmark = pytest.mark.gpu


def _sharded(wl, world, mode):
    C, D, H, W = wl["C"], wl["D"], wl["H"], wl["W"]
    runners = [parallel.SpatialRunner(wl["layers"], wl["weights"], wl["biases"], C, D, H, W, wl["brick"],
                                      wl["dtype"], r, world, mode=mode) for r in range(world)]
    x = wl["x"]
    for r, run in enumerate(runners):
        g = run.geo
        run.load(x[:, :, g.lo:g.hi].cuda())
    parallel.halo_exchange_local([r.xb for r in runners], runners[0].in_plane, [r.geo for r in runners])
    outs = [r.compute() for r in runners]
    return torch.cat(outs, dim=2).float().cpu().numpy(), runners


@pytest.mark.parametrize("world", [2, 4])
def test_spatial_sharding_bitexact_small(world):
    wl = workloads.make_workload("cfg5", D=32, H=16, W=16, C=16)
    plan = engine.plan_from_workload(wl)
    mode = plan.subgraphs()[0]["mode"]
    ref = plan.forward(wl["x"]).float().cpu().numpy()
    got, runners = _sharded(wl, world, mode)
    np.testing.assert_array_equal(got, ref)
    o = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype="bf16")
    assert float(np.max(np.abs(got - o)) / np.max(np.abs(o))) <= 2e-2


def test_spatial_sharding_full_size_8_slabs():
    """cfg5 at full size (1 x 32 x 128^3, 4^3 bricks) split into 8 slabs of 16 planes (+4 halo planes per
    interior face): the launch configuration of bench.py --config cfg5 --gpus 8."""
    wl = workloads.make_workload("cfg5")
    plan = engine.plan_from_workload(wl)
    mode = plan.subgraphs()[0]["mode"]
    ref = plan.forward(wl["x"]).float().cpu().numpy()
    got, runners = _sharded(wl, 8, mode)
    assert runners[3].geo.ext_D == 16 + 8 and runners[0].geo.ext_D == 16 + 4
    np.testing.assert_array_equal(got, ref)


def test_batch_runner_gather_on_gpu():
    """Strong-scaling runner on one GPU (world 1, NCCL when a group exists, else a copy): micro-batched merged
    execution + the gather path reproduce the one-shot plan output bit for bit, in global image order."""
    wl = workloads.make_workload("cfg4", N=4, H=64, W=64)
    plan1 = engine.plan_from_workload(wl)
    ref = plan1.forward(wl["x"])
    mb_wl = workloads.make_workload("cfg4", N=2, H=64, W=64)
    plan = engine.plan_from_workload(mb_wl)
    lo = plan.out_layout
    run = parallel.BatchRunner(4, (lo.C, lo.D, lo.H, lo.W), 0, 1, micro=2, plan=plan, device="cuda")
    x_local = wl["x"][run.global_images()].cuda().to(plan.tdtype)
    y = run.forward(x_local)
    torch.cuda.synchronize()
    assert torch.equal(y, ref)
