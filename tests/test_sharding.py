"""Spatial (D-slab) sharding of a 3-D volume with a brick-plane halo exchange:
host index logic, single-process emulation and a 2/3-rank gloo run on CPU.  The exchanged bytes are checked
against the oracle's brick layout of the whole volume (oracle/: test infrastructure only)."""
import multiprocessing as mp
import os
import socket
import sys

import numpy as np
import pytest
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_icpp_lakshminarasimhan24_b200 import parallel, workloads  # noqa: E402


def test_chain_depth_halo():
    assert parallel.chain_depth_halo(workloads.make_layers("cfg5")) == 4      # four 3x3x3 layers, p = 1
    assert parallel.chain_depth_halo(workloads.make_layers("cfg2")) == 0      # 2-D layers: k_d = 1
    with pytest.raises(ValueError):
        parallel.chain_depth_halo([workloads.conv(8, 8, k=3, s=2, nsp=3)])


@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_slab_geometry(world):
    D, Bd, halo = 128, 4, 4
    geos = [parallel.SlabGeometry(D, Bd, halo, r, world) for r in range(world)]
    assert [g.lo for g in geos] == [r * D // world for r in range(world)]
    assert geos[0].ext_lo == 0 and geos[-1].ext_lo + geos[-1].ext_D == D
    P = 1000
    for g in geos:
        assert g.ext_D == g.own + (g.lo_planes + g.hi_planes) * Bd
        for peer, snd, rcv in g.exchange_ranges(P):
            assert abs(peer - g.rank) == 1
            # what I receive from `peer` is exactly what `peer` sends to me
            back = [s for p2, s, _ in geos[peer].exchange_ranges(P) if p2 == g.rank][0]
            assert back.stop - back.start == rcv.stop - rcv.start == g.halo_planes * P
            assert snd.stop - snd.start == g.halo_planes * P


def test_slab_geometry_rejects():
    with pytest.raises(ValueError):
        parallel.SlabGeometry(128, 4, 4, 0, 3)      # 128 / 3 is not whole
    with pytest.raises(ValueError):
        parallel.SlabGeometry(16, 4, 8, 0, 4)       # halo deeper than a 4-plane slab


def _volume(D=32, H=8, W=8, C=4, seed=0):
    g = torch.Generator().manual_seed(seed)
    return torch.randn(1, C, D, H, W, generator=g, dtype=torch.float64).numpy()


def _ext_buffers(x, world, brick=(1, 4, 4, 4), halo=4, cpad=4):
    """Per-rank extended buffers holding only their own planes (halos zero) + the full-volume reference."""
    D = x.shape[2]
    full = oracle.brickify(x, brick, cpad)
    nbd = D // brick[1]
    plane = full.size // nbd
    geos = [parallel.SlabGeometry(D, brick[1], halo, r, world) for r in range(world)]
    exts = []
    for g in geos:
        e = torch.zeros(g.ext_D // brick[1] * plane, dtype=torch.float64)
        own = torch.from_numpy(full[g.lo // brick[1] * plane: g.hi // brick[1] * plane].copy())
        e[g.own_slice(plane)] = own
        exts.append(e)
    return full, plane, geos, exts


@pytest.mark.parametrize("world", [2, 4, 8])
def test_halo_exchange_local_equals_whole_volume_layout(world):
    x = _volume(D=64)
    full, plane, geos, exts = _ext_buffers(x, world)
    parallel.halo_exchange_local(exts, plane, geos)
    for g, e in zip(geos, exts):
        lo = g.ext_lo // 4 * plane
        np.testing.assert_array_equal(e.numpy(), full[lo: lo + e.numel()])


def _gloo_halo_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    x = _volume(D=48)
    full, plane, geos, exts = _ext_buffers(x, world)
    g, e = geos[rank], exts[rank]
    parallel.halo_exchange(e, plane, g)
    lo = g.ext_lo // 4 * plane
    ok = bool(np.array_equal(e.numpy(), full[lo: lo + e.numel()]))
    q.put((rank, ok))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_halo_exchange(world):
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_halo_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res == {r: True for r in range(world)}


# ---------------------------------------------------------------- batch sharding + overlapped output gather
@pytest.mark.parametrize("n,world,micro", [(256, 8, 2), (256, 2, 4), (12, 3, 2), (8, 1, 2)])
def test_micro_batches_cover_batch_in_gather_order(n, world, micro):
    mb, ranges = parallel.micro_batches(n, world, micro)
    assert mb * world * micro == n
    seen = sorted(i for r in range(world) for a, b in ranges[r] for i in range(a, b))
    assert seen == list(range(n))
    for i in range(micro):   # gathering micro-batch i rank-major gives contiguous global images
        cat = [k for r in range(world) for k in range(*ranges[r][i])]
        assert cat == list(range(i * world * mb, (i + 1) * world * mb))
    with pytest.raises(ValueError):
        parallel.micro_batches(n + 1, world, micro)


def _layer_fn(x, out):
    """Stand-in for the merged plan on CPU: one fixed conv + ReLU (the gather path is what is under test)."""
    w = torch.linspace(-1, 1, 4 * 3 * 3 * 3, dtype=torch.float64).reshape(4, 3, 3, 3)
    out.copy_(torch.relu(torch.nn.functional.conv2d(x[:, :, 0], w, padding=1))[:, :, None])
    return out


def _gloo_gather_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, micro = 4 * world, 2
    g = torch.Generator().manual_seed(5)
    x_all = torch.randn(n, 3, 1, 6, 5, generator=g, dtype=torch.float64)
    run = parallel.BatchRunner(n, (4, 1, 6, 5), rank, world, micro=micro, compute=_layer_fn, device="cpu",
                               dtype=torch.float64)
    x_local = x_all[run.global_images()].contiguous()
    y = run.forward(x_local)
    ref = _layer_fn(x_all, torch.empty(n, 4, 1, 6, 5, dtype=torch.float64))
    sharded = run.forward(x_local, gather=False)
    ok = bool(torch.equal(y, ref)) and bool(torch.equal(sharded, ref[run.global_images()]))
    q.put((rank, ok))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_batch_gather_equals_unsharded(world):
    """Strong scaling: every rank computes its micro-batches and all-gathers them; the gathered
    batch equals the unsharded computation in global image order on every rank."""
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_gather_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res == {r: True for r in range(world)}


def test_torchrun_batch_gather():
    """The multi-process launch the driver uses (python -m torch.distributed.run, env:// rendezvous on 127.0.0.1,
    one process per rank), here with 2 CPU ranks over gloo: the batch runner's all-gather equals the unsharded batch."""
    import subprocess
    import sys
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    script = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_torchrun_gather.py")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr", "127.0.0.1", "--master-port", str(port), script],
                       capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    assert "GATHER_OK" in r.stdout, r.stdout[-2000:]
