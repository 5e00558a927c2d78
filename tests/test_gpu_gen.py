"""GPU parity of the generic tcgen05 kernel (chain_tc_gen.cu) against the CPU oracle.

One graph per feature of the kernel: the three A-operand layouts (cin <= 8 tap-paired, cin % 16 chunk
planes, cin % 64 swizzled K-blocks), stride-2 polyphase tiles, 1x1 / 3x3 / 7x7 kernels, cin != cout,
several output-channel chunks, 3-D, residual epilogues, a trailing pool, ragged (non-brick-multiple)
extents.  Memoized and unmerged execution must agree bit for bit (one accumulation order per output,
SURVEY.md M4) and both must be within the bf16 tolerance of the oracle.
"""
import numpy as np
import pytest

import oracle
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads as W

pytestmark = pytest.mark.gpu
TOL = 2e-2


def rel_err(y, ref):
    y = np.asarray(y, dtype=np.float64)
    return float(np.max(np.abs(y - ref)) / max(np.max(np.abs(ref)), 1e-30))


C3 = dict(nsp=3)


def bottlenecks(cin, width, stride):
    """ResNet-50 bottleneck with a projection shortcut followed by an identity bottleneck (§4.3):
    layers read non-previous layers and add residuals produced inside the subgraph (a DAG subgraph)."""
    return [
        W.conv(cin, width, 1, inp=-1),                                   # 0
        W.conv(width, width, 3, stride),                                 # 1
        W.conv(cin, 4 * width, 1, stride, 0, relu=False, inp=-1),        # 2 projection of the block input
        W.conv(width, 4 * width, 1, inp=1, res=2, wscale=0.5),           # 3 + projection
        W.conv(4 * width, width, 1),                                     # 4
        W.conv(width, width, 3),                                         # 5
        W.conv(width, 4 * width, 1, res=3, wscale=0.5),                  # 6 + block 1 output
    ]


GRAPHS = {
    "dag_bottlenecks_s1": (bottlenecks(64, 64, 1), 2, 64, 1, 16, 16, (1, 1, 8, 8)),
    "dag_bottlenecks_s2": (bottlenecks(256, 128, 2), 2, 256, 1, 18, 14, (1, 1, 8, 8)),
    # name: (layers, N, C, D, H, W, brick)
    "pair_s1_vgg_conv1": ([W.conv(3, 64, 3)], 2, 3, 1, 20, 20, (1, 1, 8, 8)),
    "pair_s2_k7_stem": ([W.conv(3, 64, 7, 2, 3)], 2, 3, 1, 38, 38, (1, 1, 8, 8)),
    "sw128_cin_ne_cout": ([W.conv(64, 128, 3)], 2, 64, 1, 20, 20, (1, 1, 8, 8)),
    "sw128_chain_grow": ([W.conv(64, 128, 3), W.conv(128, 128, 3)], 2, 64, 1, 18, 22, (1, 1, 8, 8)),
    "bottleneck_res": ([W.conv(256, 64, 1), W.conv(64, 64, 3), W.conv(64, 256, 1, res=-1, wscale=0.5)],
                       2, 256, 1, 14, 14, (1, 1, 8, 8)),
    "s2_3x3_even": ([W.conv(64, 64, 3, 2)], 2, 64, 1, 20, 20, (1, 1, 8, 8)),
    "s2_3x3_odd": ([W.conv(128, 128, 3, 2)], 1, 128, 1, 21, 19, (1, 1, 8, 8)),
    "s2_1x1_proj": ([W.conv(256, 512, 1, 2, 0, relu=False)], 2, 256, 1, 14, 14, (1, 1, 8, 8)),
    "wide_out_nc8": ([W.conv(512, 2048, 1)], 3, 512, 1, 7, 7, (1, 1, 8, 8)),
    "planes_16_32": ([W.conv(16, 32, 3), W.conv(32, 32, 3)], 2, 16, 1, 20, 20, (1, 1, 8, 8)),
    "planes_3d": ([W.conv(32, 32, 3, nsp=3), W.conv(32, 32, 3, nsp=3)], 1, 32, 10, 12, 9, (1, 4, 4, 4)),
    # max-pool fused into the last conv's epilogue: VGG 2x2/2, ResNet stem 3x3/2 pad 1 (overlapping
    # windows: conv tiles recompute one shared row/column), ragged floor-mode extents, one conv + pool
    "pool_tail": ([W.conv(64, 64, 3), W.conv(64, 64, 3), W.pool(64, 2, 2, 0)], 2, 64, 1, 20, 20, (1, 1, 8, 8)),
    "pool_fused_2x2_ragged": ([W.conv(32, 64, 3), W.conv(64, 128, 3), W.pool(128, 2, 2, 0)], 2, 32, 1, 21, 19,
                              (1, 1, 8, 8)),
    "pool_fused_stem_3x3s2p1": ([W.conv(3, 64, 7, 2, 3), W.pool(64, 3, 2, 1)], 2, 3, 1, 38, 42, (1, 1, 8, 8)),
    "pool_fused_chain_3x3s2p1": ([W.conv(64, 64, 1), W.conv(64, 64, 3), W.pool(64, 3, 2, 1)], 2, 64, 1, 27, 30,
                                 (1, 1, 8, 8)),
    # dilated convs (DRN / DeepCAM style, L378-385): taps d apart, halo d(k-1)/2 per layer
    "dilated_chain_d2": ([W.conv(64, 64, 3, dil=2), W.conv(64, 64, 3, dil=2)], 2, 64, 1, 26, 21, (1, 1, 8, 8)),
    "dilated_mixed_d1_d3": ([W.conv(32, 64, 3), W.conv(64, 64, 3, dil=3), W.conv(64, 64, 1)], 1, 32, 1, 30, 27,
                            (1, 1, 8, 8)),
    "dilated_3d_d2": ([W.conv(32, 32, 3, nsp=3, dil=2), W.conv(32, 32, 3, nsp=3)], 1, 32, 12, 13, 10, (1, 4, 4, 4)),
    # 3x3x3 x 64 channels = 108 k-steps per layer (the Fig 10/11 microbenchmark layers)
    "sw128_3d_c64": ([W.conv(64, 64, 3, nsp=3), W.conv(64, 64, 3, nsp=3)], 1, 64, 10, 12, 9, (1, 4, 4, 4)),
    "sw128_3d_c64_valid": ([W.conv(64, 64, 3, 1, 0, nsp=3), W.conv(64, 64, 3, 1, 0, nsp=3)], 1, 64, 13, 12, 14,
                           (1, 4, 4, 4)),
    # 32-channel layers on the 64-B swizzled layout: valid padding (no stage offset) and a 1x1 layer, ragged extents
    "sw64_3d_valid_1x1": ([W.conv(32, 32, 3, 1, 0, nsp=3), W.conv(32, 32, 1, nsp=3)], 1, 32, 11, 13, 14,
                          (1, 4, 4, 4)),
    "sw64_2d_chain": ([W.conv(32, 64, 3), W.conv(64, 32, 1)], 2, 32, 1, 19, 21, (1, 1, 8, 8)),
}


@pytest.mark.parametrize("fuse", [0, 1])
@pytest.mark.parametrize("name", sorted(GRAPHS))
def test_gen_vs_oracle(name, fuse):
    layers, N, C, D, H, Wd, brick = GRAPHS[name]
    nsp = 3 if brick[1] > 1 else 2
    wl = W.make_graph_workload(layers, N, C, D, H, Wd, nsp, brick, "bf16", seed=11)
    ref = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype="bf16")
    plan = engine.plan_from_workload(wl, force_mode=2, fuse_pool=fuse)
    sgs = plan.subgraphs()
    assert any(s["kernel"] == "tcgen05 generic" for s in sgs), sgs
    outs = {}
    for mode in ("memoized", "unmerged", "padded"):
        plan.set_mode(mode)
        outs[mode] = plan.forward(wl["x"]).float().cpu().numpy()
        assert rel_err(outs[mode], ref) <= TOL, (mode, rel_err(outs[mode], ref))
    np.testing.assert_array_equal(outs["memoized"], outs["unmerged"])
    np.testing.assert_array_equal(outs["memoized"], outs["padded"])
    plan.set_mode("memoized")
    plan.forward(wl["x"])
    for i, s in enumerate(sgs):
        nconv = sum(l["kind"] == "conv" for l in wl["layers"][s["first"]:s["last"] + 1])
        if s["kernel"] == "tcgen05 generic" and nconv > 1:
            c = plan.counters(i)
            assert c["computed"] == c["cas_ok"] and c["computed"] > 0, c


@pytest.mark.parametrize("brick", [4, 8, 16, 64])
def test_gen_padded_block_sizes(brick):
    """Padded mode with blocks of several edges (regions of edge, interior and single-block images):
    every block recomputes its halo (§3.2.1, Fig 4) and matches memoized execution exactly."""
    layers = [W.conv(64, 64, 3), W.conv(64, 128, 1), W.conv(128, 64, 3, res=-1, wscale=0.5)]
    wl = W.make_graph_workload(layers, 2, 64, 1, 30, 27, 2, (1, 1, 8, 8), "bf16", seed=3)
    ref = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype="bf16")
    plan = engine.plan_from_workload(wl, force_mode=1, force_brick=brick)
    assert plan.subgraphs()[0]["kernel"] == "tcgen05 generic" and plan.subgraphs()[0]["last"] == 2
    yp = plan.forward(wl["x"]).float().cpu().numpy()
    assert rel_err(yp, ref) <= TOL
    for _ in range(3):   # repeated runs: ticket accounting across launches
        np.testing.assert_array_equal(plan.forward(wl["x"]).float().cpu().numpy(), yp)
    plan.set_mode("memoized")
    ym = plan.forward(wl["x"]).float().cpu().numpy()
    np.testing.assert_array_equal(yp, ym)


def test_gen_repeat_and_masking():
    """Repeated runs reuse the memo table through epoch tags; masked (out-of-image) positions of the
    bricked output are zero."""
    layers = [W.conv(64, 128, 3), W.conv(128, 64, 1, res=-1, wscale=0.5)]
    wl = W.make_graph_workload(layers, 2, 64, 1, 13, 11, 2, (1, 1, 8, 8), "bf16", seed=5)
    plan = engine.plan_from_workload(wl, force_mode=2)
    xb = plan.brickify(wl["x"])
    yb = plan.run(xb)
    first = yb.clone()
    for _ in range(3):
        assert bool((plan.run(xb) == first).all())
    # bricked output: bricks of 8x8 x 64 ch; image 13 x 11 -> grid 16 x 16; masked pixels must be 0
    import torch
    v = first.view(torch.bfloat16).view(2, 2, 2, 8, 8, 64).float()   # [n][by][bx][y][x][c]
    full = v.permute(0, 1, 3, 2, 4, 5).reshape(2, 16, 16, 64)
    assert float(full[:, 13:].abs().max()) == 0.0 and float(full[:, :, 11:].abs().max()) == 0.0


def test_dag_subgraph_schedule_invariance():
    """A bottleneck DAG (projection + identity block) as ONE merged memoized subgraph: any task order gives
    bit-identical results with every task computed exactly once (computed == successful claims: 2 compulsory
    atomics per task, L1147-1149; merged execution only reorders work, L363-365).  Seeds select random
    topological orders; seed 0 is the locality-aware wavefront."""
    layers, N, C, D, H, Wd, brick = GRAPHS["dag_bottlenecks_s1"]
    wl = W.make_graph_workload(layers, N, C, D, H, Wd, 2, brick, "bf16", seed=17)
    ref = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype="bf16")
    y0, n0 = None, None
    # memo_defer=1: the paper's "move on and revisit" hand-over (claimed tasks with in-progress dependencies are
    # set aside); 0: in-order hand-over, the loader waits
    for seed, defer in ((0, 0), (0, 1), (1, 0), (7, 1), (123, 0), (123, 1)):
        plan = engine.plan_from_workload(wl, force_mode=2, schedule_seed=seed, memo_defer=defer)
        sgs = plan.subgraphs()
        assert len(sgs) == 1 and sgs[0]["mode"] == "memoized" and sgs[0]["kernel"] == "tcgen05 generic", sgs
        y = plan.forward(wl["x"]).float().cpu().numpy()
        c = plan.counters(0)
        assert c["computed"] == c["cas_ok"] and c["computed"] > 0, (seed, defer, c)
        if y0 is None:
            y0, n0 = y, c["computed"]
            assert rel_err(y, ref) <= TOL
        else:
            np.testing.assert_array_equal(y, y0)
            assert c["computed"] == n0
    plan.set_mode("unmerged")
    np.testing.assert_array_equal(plan.forward(wl["x"]).float().cpu().numpy(), y0)


@pytest.mark.parametrize("which", ["band_cfg2", "gen_dag"])
def test_cuda_graph_replay(which):
    """The per-run memo state (ticket counter, tag epoch) lives on the device, so a captured bdl_run replays
    correctly: each replay recomputes from its current input."""
    import torch
    if which == "band_cfg2":
        wl = W.make_workload("cfg2", N=2, H=24, W=24)
    else:
        layers, N, C, D, H, Wd, brick = GRAPHS["dag_bottlenecks_s1"]
        wl = W.make_graph_workload(layers, N, C, D, H, Wd, 2, brick, "bf16", seed=19)
    plan = engine.plan_from_workload(wl, force_mode=2)
    xs = [wl["x"], (wl["x"] * -0.5).to(torch.bfloat16).float(), (wl["x"] + 0.25).to(torch.bfloat16).float()]
    refs = [plan.forward(x).clone() for x in xs]
    xb = plan.brickify(xs[0])
    yb = plan.alloc_bricked(plan.out_layout)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        plan.run(xb, yb)
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        plan.run(xb, yb)
    for rep in range(2):
        for x, ref in zip(xs, refs):
            plan.brickify(x, out=xb)
            g.replay()
            y = plan.unbrickify(yb)
            torch.cuda.synchronize()
            assert torch.equal(y, ref), (which, rep)


@pytest.mark.parametrize("brick", [4, 8, 16])
def test_gen_padded_fused_pool_blocks(brick):
    """Padded mode with the pool fused into the last conv: each block's pooled region maps back through the pool
    window (Fig 4 with the pool stride as padding factor, L456-458) and the chain; several block edges."""
    layers = [W.conv(64, 64, 3), W.conv(64, 64, 3), W.pool(64, 3, 2, 1)]
    wl = W.make_graph_workload(layers, 2, 64, 1, 30, 27, 2, (1, 1, 8, 8), "bf16", seed=23)
    ref = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype="bf16")
    plan = engine.plan_from_workload(wl, force_mode=1, force_brick=brick, fuse_pool=1)
    assert plan.subgraphs()[0]["last"] == 2 and plan.launches_per_run == 1   # one launch: the pool is fused
    yp = plan.forward(wl["x"]).float().cpu().numpy()
    assert rel_err(yp, ref) <= TOL
    plan.set_mode("memoized")
    np.testing.assert_array_equal(plan.forward(wl["x"]).float().cpu().numpy(), yp)
    # the separate pool kernel (fuse_pool=2) gives the same bits
    p2 = engine.plan_from_workload(wl, force_mode=1, force_brick=brick, fuse_pool=2)
    assert p2.launches_per_run == 2
    np.testing.assert_array_equal(p2.forward(wl["x"]).float().cpu().numpy(), yp)


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_grouped_and_depthwise(dtype):
    """Grouped and depthwise convs (MobileNet-style separable block: depthwise 3x3 -> pointwise 1x1; L378-385) run on
    the CUDA-core brick kernels (not a dense contraction); bf16 graphs cut the subgraph between the depthwise and the
    dense layers so the pointwise convs stay on the tensor cores.  Every mode against the oracle."""
    layers = [W.conv(32, 32, 3, groups=32), W.conv(32, 64, 1), W.conv(64, 64, 3, groups=8),
              W.conv(64, 64, 3, groups=64, dil=2), W.conv(64, 32, 1, res=None)]
    wl = W.make_graph_workload(layers, 2, 32, 1, 19, 22, 2, (1, 1, 8, 8), dtype, seed=29)
    ref = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype=dtype)
    plan = engine.plan_from_workload(wl, force_mode=2)
    sgs = plan.subgraphs()
    if dtype == "bf16":
        kinds = {(s["first"], s["last"]): s["kernel"] for s in sgs}
        assert any(k == "tcgen05 generic" for k in kinds.values()), kinds      # the pointwise convs
        assert any(k == "cuda-core brick" for k in kinds.values()), kinds      # the depthwise / grouped convs
    outs = {}
    for mode in ("memoized", "padded", "unmerged"):
        plan.set_mode(mode)
        outs[mode] = plan.forward(wl["x"]).float().cpu().numpy()
        assert rel_err(outs[mode], ref) <= (TOL if dtype == "bf16" else 1e-5), (mode, rel_err(outs[mode], ref))
    np.testing.assert_array_equal(outs["memoized"], outs["unmerged"])
    np.testing.assert_array_equal(outs["memoized"], outs["padded"])


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_transposed_conv_chain(dtype):
    """Transposed convs (the last of the L378-385 mergeable ops): an encoder-decoder chain -- 3x3 stride-2 conv down,
    2x upsampling transposed conv (k 4, s 2, p 1), a dilated stride-1 transposed conv, a 3x3 conv with the graph input
    as residual -- runs on the CUDA-core brick kernels (bf16: the dense convs stay on the tensor cores); every mode
    against the oracle, the merged modes bit-equal to unmerged."""
    layers = [W.conv(16, 32, 3, s=2), W.conv(32, 16, 4, s=2, transposed=True), W.conv(16, 16, 3, dil=2, transposed=True),
              W.conv(16, 16, 3, res=-1, wscale=0.5)]
    wl = W.make_graph_workload(layers, 2, 16, 1, 20, 24, 2, (1, 1, 8, 8), dtype, seed=31)
    assert tuple(wl["x"].shape[-2:]) == (20, 24)
    ref = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype=dtype)
    assert ref.shape[-2:] == (20, 24)
    plan = engine.plan_from_workload(wl, force_mode=2)
    if dtype == "bf16":
        kinds = {s["kernel"] for s in plan.subgraphs()}
        assert "cuda-core brick" in kinds and "tcgen05 generic" in kinds, kinds
    outs = {}
    for mode in ("memoized", "padded", "unmerged"):
        plan.set_mode(mode)
        outs[mode] = plan.forward(wl["x"]).float().cpu().numpy()
        assert rel_err(outs[mode], ref) <= (TOL if dtype == "bf16" else 1e-5), (mode, rel_err(outs[mode], ref))
    np.testing.assert_array_equal(outs["memoized"], outs["unmerged"])
    np.testing.assert_array_equal(outs["memoized"], outs["padded"])
