"""CPU tests of the C ABI library and its host logic (no device work): symbol exports, layout
geometry, BrickInfo (Fig 6), region analysis (Fig 4), the rho/tau brick model, the Delta mode rule,
graph partitioning invariants, and batch sharding under a 2-process gloo group."""
import ctypes
import json
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_icpp_lakshminarasimhan24_b200 as bdl
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, parallel, workloads

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_icpp_lakshminarasimhan24_b200 import build
    build.build()


def test_library_exports_every_header_symbol():
    hdr = open(os.path.join(ROOT, "include", "brickdl.h")).read()
    declared = set(re.findall(r"\b(bdl_[a-z_]+)\s*\(", hdr))
    assert len(declared) >= 20
    L = bdl.lib()
    for name in sorted(declared):
        assert hasattr(L, name), name
        assert name in bdl.EXPORTS, f"binding lacks {name}"
    assert bdl.lib().bdl_version().startswith(b"brickdl")


@pytest.mark.parametrize("args,nb,cpad", [
    ((2, 1, 8, 1, 32, 32, 1, 1, 8, 8, bdl.BDL_F32), (1, 1, 4, 4), 8),
    ((2, 64, 64, 1, 56, 56, 1, 1, 8, 8, bdl.BDL_BF16), (64, 1, 7, 7), 64),
    ((2, 3, 3, 1, 224, 224, 2, 1, 16, 16, bdl.BDL_BF16), (2, 1, 14, 14), 8),
    ((3, 1, 32, 128, 128, 128, 1, 4, 4, 4, bdl.BDL_BF16), (1, 32, 32, 32), 32),
    ((2, 5, 5, 1, 7, 9, 1, 1, 4, 4, bdl.BDL_F32), (5, 1, 2, 3), 8),
])
def test_layout_init(args, nb, cpad):
    lo = engine.make_layout(args[0], *args[1:6], args[6:10], args[10])
    assert tuple(lo.nb) == nb and lo.c_pad == cpad
    assert lo.nbricks == np.prod(nb)
    assert lo.brick_elems == np.prod(args[6:10]) * cpad
    assert lo.total_bytes == lo.nbricks * lo.brick_elems * (4 if args[10] == bdl.BDL_F32 else 2)


def test_layout_init_errors():
    lo = bdl.bdl_layout()
    assert bdl.lib().bdl_layout_init(ctypes.byref(lo), 2, 1, 8, 2, 32, 32, 1, 1, 8, 8, 0) == bdl.BDL_EINVAL
    assert b"D = 1" in bdl.lib().bdl_last_error()
    assert bdl.lib().bdl_layout_init(ctypes.byref(lo), 2, 0, 8, 1, 32, 32, 1, 1, 8, 8, 0) == bdl.BDL_EINVAL
    assert bdl.lib().bdl_layout_init(ctypes.byref(lo), 4, 1, 8, 1, 32, 32, 1, 1, 8, 8, 0) == bdl.BDL_EINVAL
    assert bdl.lib().bdl_layout_init(ctypes.byref(lo), 2, 1, 8, 1, 32, 32, 1, 1, 8, 8, 7) == bdl.BDL_EINVAL


def _brickinfo(nsp, grid, bm=None):
    nbd, nbh, nbw = grid
    lo = engine.make_layout(nsp, 1, 4, nbd * 4 if nsp == 3 else 1, nbh * 4, nbw * 4,
                            (1, 4 if nsp == 3 else 1, 4, 4), bdl.BDL_F32)
    ndir = (27 if nsp == 3 else 9) - 1
    adj = np.empty((nbd * nbh * nbw, ndir), dtype=np.int32)
    bmp = None
    if bm is not None:
        bm = np.ascontiguousarray(bm, dtype=np.int32)
        bmp = bm.ctypes.data_as(ctypes.c_void_p)
    bdl.check(bdl.lib().bdl_brickinfo(ctypes.byref(lo), bmp, adj.ctypes.data_as(ctypes.c_void_p)))
    return adj


def test_brickinfo_fig6():
    g = json.load(open(os.path.join(GOLDEN, "fig6_brickinfo.json")))
    bm = np.array(g["brickmap"], dtype=np.int32).reshape(-1)
    adj = _brickinfo(2, (1, 4, 4), bm)
    assert adj[0].tolist() == g["eta_phys0"]


@pytest.mark.parametrize("nsp,grid", [(2, (1, 5, 3)), (3, (3, 2, 4))])
def test_brickinfo_matches_oracle(nsp, grid):
    rng = np.random.default_rng(5)
    bm = rng.permutation(int(np.prod(grid))).astype(np.int32)
    np.testing.assert_array_equal(_brickinfo(nsp, grid, bm), oracle.brickinfo(nsp, grid, bm))


def test_brickinfo_rejects_non_permutation():
    lo = engine.make_layout(2, 1, 4, 1, 8, 8, (1, 1, 4, 4), bdl.BDL_F32)
    bm = np.array([0, 0, 1, 2], dtype=np.int32)
    adj = np.empty((4, 8), dtype=np.int32)
    st = bdl.lib().bdl_brickinfo(ctypes.byref(lo), bm.ctypes.data_as(ctypes.c_void_p), adj.ctypes.data_as(ctypes.c_void_p))
    assert st == bdl.BDL_EINVAL


# ------------------------------------------------------------------------------ static analysis
def _layers(specs):
    arr = (bdl.bdl_layer * len(specs))()
    for i, (kind, k, s, p) in enumerate(specs):
        a = arr[i]
        a.kind = kind
        a.cin = a.cout = 8
        a.k[:] = [1, k, k]
        a.stride[:] = [1, s, s]
        a.pad[:] = [0, p, p]
        a.input = i - 1
        a.residual = bdl.BDL_NO_RESIDUAL
    return arr


def _regions(specs, b, dim=2):
    arr = _layers(specs)
    out = (ctypes.c_int64 * len(specs))()
    bdl.check(bdl.lib().bdl_region_extents(arr, 0, len(specs) - 1, dim, b, out))
    return list(out)


def test_region_fig4_two_convs():
    # Fig 4 (L443-455): an output brick B needs B+4p input and a B+2p intermediate (p = 1 for 3x3)
    assert _regions([(0, 3, 1, 1), (0, 3, 1, 1)], 8) == [12, 10]
    assert _regions([(0, 5, 1, 2), (0, 5, 1, 2)], 8) == [16, 12]
    # elementwise-like 1x1: no padding (L455-456)
    assert _regions([(0, 1, 1, 0), (0, 1, 1, 0)], 8) == [8, 8]
    # max pool with stride Sp: B x Sp (L456-458)
    assert _regions([(0, 3, 1, 1), (1, 2, 2, 0)], 8) == [18, 16]


def test_rho_tau_model_reproduces_paper_choices():
    rho = ctypes.c_int64()
    # L1396: 112^3 microbenchmark uses 8^3 bricks;  L1534: 224^3 best with 16^3 (tau = 2^12)
    assert bdl.lib().bdl_model_brick(None, 3, 1, 112, 112, 112, ctypes.byref(rho)) == 8
    assert rho.value == 2744
    assert bdl.lib().bdl_model_brick(None, 3, 1, 224, 224, 224, ctypes.byref(rho)) == 16
    # cfg2 (N=64, 56x56): 64*56*56/8^2 = 3136 <= 4096
    assert bdl.lib().bdl_model_brick(None, 2, 64, 1, 56, 56, ctypes.byref(rho)) == 8


def _plan(cfg, **kw):
    c = dict(workloads.CONFIGS[cfg])
    c.update(kw)
    L = workloads.make_layers(cfg, C=c["C"])
    return engine.Plan(L, None, None, c["N"], c["C"], c["D"], c["H"], c["W"], c["nsp"], c["dtype"],
                       c["brick"], device=None)


def test_delta_hand_computed():
    # 2 x conv3x3 over a 16x16 map in 8x8 bricks.  Per dim, layer-2 input regions clip to 9 + 9 = 18,
    # layer-1 input to 10 + 10 = 20, halo-free 16:  Delta = (20^2 + 18^2) / (2 * 16^2) - 1.
    p = _plan("cfg1", N=1, H=16, W=16)
    sg = p.subgraphs()[0]
    assert sg["delta"] == pytest.approx((400 + 324) / 512 - 1, abs=1e-12)
    assert sg["delta_first"] == pytest.approx(400 / 256 - 1, abs=1e-12)


def test_mode_rule_delta_threshold():
    # Delta > 15% -> memoized (L644); cfg2 at 8x8 bricks has Delta ~ 0.76
    sg = _plan("cfg2").subgraphs()[0]
    assert sg["delta"] > 0.15 and sg["mode"] == "memoized" and sg["kernel"] == "tcgen05 band"
    # 1x1 convs have no halo: Delta = 0 -> padded
    L = [dict(kind="conv", cin=8, cout=8, k=(1, 1, 1), stride=(1, 1, 1), pad=(0, 0, 0), relu=True,
              input=i - 1, residual=None, wscale=1.0) for i in range(3)]
    p = engine.Plan(L, None, None, 4, 8, 1, 64, 64, 2, "f32", (1, 1, 8, 8), device=None)
    sg = p.subgraphs()[0]
    assert sg["delta"] == 0 and sg["mode"] == "padded"


def test_tiny_layer_rule_unmerged():
    # rho < B^n -> library (here: single-layer) execution (L659-662): cfg1 at 8x8 bricks, rho = 16 < 64
    sg = _plan("cfg1").subgraphs()[0]
    assert sg["rho"] == 64 and sg["mode"] == "unmerged"


@pytest.mark.parametrize("cfg", ["cfg3", "cfg4"])
def test_partition_invariants(cfg):
    """Reverse-traversal partition (L603-626): subgraphs tile the layer list, pools end subgraphs, every layer
    reads a layer of its own subgraph or a materialized earlier one, and branched subgraphs (projection
    shortcuts, residuals produced inside, inner live-outs) run memoized on the generic tcgen05 kernel."""
    p = _plan(cfg, N=2)
    L = workloads.make_layers(cfg)
    sgs = p.subgraphs()
    covered = []
    for sg in sgs:
        f, e = sg["first"], sg["last"]
        covered += list(range(f, e + 1))
        assert e - f + 1 <= 16
        branched = False
        for j in range(f, e + 1):
            if j < e:
                assert L[j]["kind"] != "maxpool"            # pools end subgraphs (L620-626)
            assert L[j]["input"] < j                         # producers come first (topological listing)
            r = L[j]["residual"]
            branched |= (j > f and L[j]["input"] != j - 1) or (r is not None and r >= f)
            branched |= j < e and any(L[m]["input"] == j or L[m]["residual"] == j for m in range(e + 1, len(L)))
        if branched:
            assert sg["mode"] in ("memoized", "unmerged") and sg["kernel"] == "tcgen05 generic"
    assert covered == list(range(len(L)))
    if cfg == "cfg3":
        pools = [i for i, l in enumerate(L) if l["kind"] == "maxpool"]
        ends = {sg["last"] for sg in sgs}
        assert all(pi in ends for pi in pools)
        assert all(sg["first"] < sg["last"] for sg in sgs)   # no pool-only subgraph
    if cfg == "cfg4":
        # the paper splits ResNet-50 into 7 merged subgraphs (L1130-1165); we allow branches inside subgraphs,
        # so no projection or pool runs alone
        assert len(sgs) <= 10
        assert all(sg["first"] < sg["last"] for sg in sgs)


def test_partition_chain_only_for_cuda_core_path():
    """fp32 graphs run on the CUDA-core brick kernels, which merge chains only: branches cut subgraphs."""
    L = workloads.make_layers("cfg4")[:9]
    p = engine.Plan(L, None, None, 1, 3, 1, 64, 64, 2, "f32", (1, 1, 8, 8), device=None)
    for sg in p.subgraphs():
        for j in range(sg["first"] + 1, sg["last"] + 1):
            assert L[j]["input"] == j - 1
            r = L[j]["residual"]
            assert r is None or r < sg["first"]


def test_plan_opts_force_mode_and_budget():
    o = engine.default_opts(force_mode=bdl.BDL_MODE_PADDED)
    c = workloads.CONFIGS["cfg2"]
    p = engine.Plan(workloads.make_layers("cfg2"), None, None, 64, 64, 1, 56, 56, 2, "bf16", c["brick"],
                    opts=o, device=None)
    assert p.subgraphs()[0]["mode"] == "padded"
    # a tiny on-chip budget forbids merging (L611-614): every layer becomes its own subgraph
    o2 = engine.default_opts(onchip_budget=1024)
    p2 = engine.Plan(workloads.make_layers("cfg2"), None, None, 64, 64, 1, 56, 56, 2, "bf16", c["brick"],
                     opts=o2, device=None)
    assert p2.num_subgraphs == 2


def test_partition_rejects_bad_graph():
    L = workloads.make_layers("cfg1")
    L[1] = dict(L[1], cin=4)
    with pytest.raises(bdl.BrickDLError):
        engine.Plan(L, None, None, 1, 8, 1, 32, 32, 2, "f32", (1, 1, 8, 8), device=None)


# ------------------------------------------------------------------------------ sharding (gloo)
def test_shard_ranges():
    for n, w in [(64, 1), (64, 8), (256, 3), (5, 8)]:
        ranges = [parallel.shard(n, r, w) for r in range(w)]
        assert ranges[0][0] == 0 and ranges[-1][1] == n
        assert all(a[1] == b[0] for a, b in zip(ranges, ranges[1:]))
        assert max(h - l for l, h in ranges) - min(h - l for l, h in ranges) <= 1


def _gloo_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    lo, hi = parallel.shard(37, rank, world)
    mine = torch.arange(lo, hi, dtype=torch.int64)
    sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(sizes, torch.tensor([hi - lo]))
    padded = torch.full((int(max(s.item() for s in sizes)),), -1, dtype=torch.int64)
    padded[: hi - lo] = mine
    out = [torch.empty_like(padded) for _ in range(world)]
    dist.all_gather(out, padded)
    t = torch.tensor([float(rank + 1)])
    dist.all_reduce(t, op=dist.ReduceOp.MAX)    # bench.py's max-over-ranks timing reduction
    if rank == 0:
        got = torch.cat([o[o >= 0] for o in out]).tolist()
        q.put((got, t.item()))
    dist.destroy_process_group()


def test_gloo_two_ranks_cover_batch_once():
    import multiprocessing as mp
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got, tmax = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
    assert got == list(range(37)) and tmax == 2.0


# ------------------------------------------------------------------------------ transposed convolution regions
def _tlayers(specs):
    """specs: (k, s, p, d, transposed) per layer, 8 channels, a chain along the listing."""
    arr = (bdl.bdl_layer * len(specs))()
    for i, (k, s, p, d, tr) in enumerate(specs):
        a = arr[i]
        a.kind = bdl.BDL_OP_CONV
        a.cin = a.cout = 8
        a.k[:] = [1, k, k]
        a.stride[:] = [1, s, s]
        a.pad[:] = [0, p, p]
        a.dil[:] = [1, d, d]
        a.input = i - 1
        a.residual = bdl.BDL_NO_RESIDUAL
        a.transposed = tr
    return arr


def _tregions(specs, b):
    out = (ctypes.c_int64 * len(specs))()
    bdl.check(bdl.lib().bdl_region_extents(_tlayers(specs), 0, len(specs) - 1, 2, b, out))
    return list(out)


@pytest.mark.parametrize("k,s,p,d", [(4, 2, 1, 1), (2, 2, 0, 1), (3, 2, 1, 1), (3, 1, 1, 2), (5, 3, 2, 1)])
def test_region_transposed_brute_force(k, s, p, d):
    """Reverse traversal through a transposed conv: the input region of an output brick [0, b) is the hull of the
    inputs i with s*i - p + d*t in [0, b) for some tap t (enumerated here)."""
    for b in (4, 8, 16):
        reach = [i for i in range(-4 * b, 4 * b) if any(0 <= s * i - p + d * t < b for t in range(k))]
        assert _tregions([(k, s, p, d, 1)], b) == [max(reach) - min(reach) + 1]


def test_region_chain_through_transposed():
    # 3x3 conv (p = 1) then a 2x upsampling transposed conv (k 4, s 2, p 1): brick 8 of the output needs inputs
    # [-1, 4] of the transposed conv (6) and 6 + 2 of the first conv
    assert _tregions([(3, 1, 1, 1, 0), (4, 2, 1, 1, 1)], 8) == [8, 6]
