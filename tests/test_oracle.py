"""Pins of the CPU oracle against what the paper and the mathematics fix.

Each test pins the oracle to something other than itself: closed forms (P1-P3), a composed-kernel
identity that exposes the Fig 4 halo growth and the zero-padded intermediate (P4), brute force by
an independently assembled dense operator (P5), a library routine (P6, torch fp64), an invariance
(P7), torch's own bf16 cast, and the paper's Fig 6 worked example.
"""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_icpp_lakshminarasimhan24_b200 import workloads

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
rng = np.random.default_rng(12345)


# ---------------------------------------------------------------- P1 delta input (orientation)
@pytest.mark.parametrize("stride,pad,k", [(1, 1, 3), (2, 1, 3), (1, 0, 3), (2, 3, 7), (1, 0, 1)])
def test_p1_delta_input_2d(stride, pad, k):
    N, C, H, W, Co = 2, 3, 9, 11, 4
    n0, c0, h0, w0 = 1, 2, 4, 5
    x = np.zeros((N, C, H, W))
    x[n0, c0, h0, w0] = 1.0
    w = rng.standard_normal((Co, C, k, k))
    y = oracle.conv(x, w, stride=(stride, stride), pad=(pad, pad))
    Ho, Wo = y.shape[2:]
    expect = np.zeros_like(y)
    # y[n0, co, oh, ow] = w[co, c0, r, s] where stride*oh - pad + r = h0 (cross-correlation)
    for oh in range(Ho):
        for ow in range(Wo):
            r = h0 - (stride * oh - pad)
            s = w0 - (stride * ow - pad)
            if 0 <= r < k and 0 <= s < k:
                expect[n0, :, oh, ow] = w[:, c0, r, s]
    np.testing.assert_array_equal(y, expect)


def test_p1_delta_input_3d():
    N, C, D, H, W, Co, k, p = 1, 2, 6, 5, 7, 3, 3, 1
    x = np.zeros((N, C, D, H, W))
    x[0, 1, 2, 3, 4] = 1.0
    w = rng.standard_normal((Co, C, k, k, k))
    y = oracle.conv(x, w, stride=(1, 1, 1), pad=(p, p, p))
    expect = np.zeros_like(y)
    for r in range(k):
        for s in range(k):
            for t in range(k):
                od, oh, ow = 2 + p - r, 3 + p - s, 4 + p - t
                if 0 <= od < D and 0 <= oh < H and 0 <= ow < W:
                    expect[0, :, od, oh, ow] = w[:, 1, r, s, t]
    np.testing.assert_array_equal(y, expect)


# ---------------------------------------------------------------- P2 identity kernel
def _identity_w(C, k=3, nsp=2):
    if nsp == 2:
        w = np.zeros((C, C, 1, k, k))
        for c in range(C):
            w[c, c, 0, k // 2, k // 2] = 1.0
    else:
        w = np.zeros((C, C, k, k, k))
        for c in range(C):
            w[c, c, k // 2, k // 2, k // 2] = 1.0
    return w


def test_p2_identity_chain_relu_and_residual():
    C, L = 4, 3
    x = rng.standard_normal((2, C, 1, 10, 9))
    layers = workloads.make_layers("cfg1", C=C, nlayers=L)
    ws = [_identity_w(C)] * L
    bs = [np.zeros(C)] * L
    y = oracle.run_graph(layers, x, ws, bs, dtype="f64")
    np.testing.assert_array_equal(y, np.maximum(x, 0))
    # cfg2 graph: conv-relu, conv + x, relu  ->  relu(relu(x) + x) = 2 relu(x)
    layers2 = workloads.make_layers("cfg2", C=C)
    y2 = oracle.run_graph(layers2, x, [_identity_w(C)] * 2, [np.zeros(C)] * 2, dtype="f64")
    np.testing.assert_array_equal(y2, 2 * np.maximum(x, 0))


# ---------------------------------------------------------------- P3 border counts
def test_p3_ones_border_counts_2d():
    C, b = 5, 0.25
    x = np.ones((1, C, 6, 7))
    w = np.ones((2, C, 3, 3))
    y = oracle.conv(x, w, bias=np.full(2, b), pad=(1, 1))
    assert y[0, 0, 3, 3] == C * 9 + b      # interior
    assert y[0, 1, 0, 3] == C * 6 + b      # edge
    assert y[0, 0, 3, 6] == C * 6 + b
    assert y[0, 0, 0, 0] == C * 4 + b      # corner
    assert y[0, 0, 5, 6] == C * 4 + b


def test_p3_ones_border_counts_3d():
    C = 2
    x = np.ones((1, C, 5, 5, 5))
    y = oracle.conv(x, np.ones((1, C, 3, 3, 3)), pad=(1, 1, 1))
    assert y[0, 0, 2, 2, 2] == C * 27
    assert y[0, 0, 0, 2, 2] == C * 18      # face
    assert y[0, 0, 0, 0, 2] == C * 12      # edge
    assert y[0, 0, 0, 0, 0] == C * 8       # corner


# ---------------------------------------------------------------- P4 composed kernel / Fig 4
def test_p4_composed_kernel_interior_and_zero_padded_intermediate():
    """Two bias-free 3x3 convs equal one 5x5 conv with the composed kernel in the interior, i.e. an
    output brick needs a (B+4p) input region (Fig 4).  Within 2p of the border they
    DIFFER because the intermediate is zero-padded, not recomputed."""
    C, H, W = 3, 12, 13
    x = rng.standard_normal((1, C, H, W))
    w1 = rng.standard_normal((C, C, 3, 3))
    w2 = rng.standard_normal((C, C, 3, 3))
    y2 = oracle.conv(oracle.conv(x, w1, pad=(1, 1)), w2, pad=(1, 1))
    # composed kernel K[o,i,u,v] = sum_m sum_{r+r'=u, s+s'=v} w2[o,m,r,s] w1[m,i,r',s']
    K = np.zeros((C, C, 5, 5))
    for r in range(3):
        for s in range(3):
            for r2 in range(3):
                for s2 in range(3):
                    K[:, :, r + r2, s + s2] += w2[:, :, r, s] @ w1[:, :, r2, s2]
    yc = oracle.conv(x, K, pad=(2, 2))
    np.testing.assert_allclose(y2[..., 2:-2, 2:-2], yc[..., 2:-2, 2:-2], rtol=1e-12, atol=1e-12)
    border = np.ones((H, W), bool)
    border[2:-2, 2:-2] = False
    assert np.max(np.abs(y2[..., border] - yc[..., border])) > 1e-3


# ---------------------------------------------------------------- P5 brute force dense operator
def _dense_conv_operator(Ci, Co, H, W, w, stride, pad):
    k = w.shape[-1]
    Ho = (H + 2 * pad - k) // stride + 1
    Wo = (W + 2 * pad - k) // stride + 1
    T = np.zeros((Co * Ho * Wo, Ci * H * W))
    for co in range(Co):
        for oh in range(Ho):
            for ow in range(Wo):
                row = (co * Ho + oh) * Wo + ow
                for ci in range(Ci):
                    for ih in range(H):
                        for iw in range(W):
                            r, s = ih - (stride * oh - pad), iw - (stride * ow - pad)
                            if 0 <= r < k and 0 <= s < k:
                                T[row, (ci * H + ih) * W + iw] = w[co, ci, r, s]
    return T, Ho, Wo


@pytest.mark.parametrize("stride,pad", [(1, 1), (2, 1), (1, 0)])
def test_p5_bruteforce_dense(stride, pad):
    N, Ci, Co, H, W = 2, 3, 2, 7, 6
    x = rng.standard_normal((N, Ci, H, W))
    w = rng.standard_normal((Co, Ci, 3, 3))
    T, Ho, Wo = _dense_conv_operator(Ci, Co, H, W, w, stride, pad)
    y = oracle.conv(x, w, stride=(stride, stride), pad=(pad, pad))
    for n in range(N):
        np.testing.assert_allclose(y[n].reshape(-1), T @ x[n].reshape(-1), rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- P6 library routine (torch fp64)
@pytest.mark.parametrize("k,s,p", [(3, 1, 1), (3, 2, 1), (7, 2, 3), (1, 1, 0), (1, 2, 0)])
def test_p6_torch_conv2d(k, s, p):
    x = rng.standard_normal((2, 5, 13, 11))
    w = rng.standard_normal((6, 5, k, k))
    b = rng.standard_normal(6)
    y = oracle.conv(x, w, bias=b, stride=(s, s), pad=(p, p))
    ref = torch.nn.functional.conv2d(torch.from_numpy(x), torch.from_numpy(w), torch.from_numpy(b),
                                     stride=s, padding=p).numpy()
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


def test_p6_torch_conv3d():
    x = rng.standard_normal((1, 3, 6, 7, 5))
    w = rng.standard_normal((4, 3, 3, 3, 3))
    y = oracle.conv(x, w, pad=(1, 1, 1))
    ref = torch.nn.functional.conv3d(torch.from_numpy(x), torch.from_numpy(w), padding=1).numpy()
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("k,s,p", [(2, 2, 0), (3, 2, 1)])
def test_p6_torch_maxpool(k, s, p):
    x = rng.standard_normal((2, 3, 11, 12))
    y = oracle.maxpool(x, (1, k, k), (1, s, s), (0, p, p))
    ref = torch.nn.functional.max_pool2d(torch.from_numpy(x), k, s, p).numpy()
    np.testing.assert_array_equal(y, ref)


def test_p6_chain_vs_torch():
    wl = workloads.make_workload("cfg2", N=2, C=8, H=11, W=9)
    x = wl["x"].double()[:, :, 0]
    w = [t.double()[:, :, 0] for t in wl["weights"]]
    b = [t.double() for t in wl["biases"]]
    F = torch.nn.functional
    h = torch.relu(F.conv2d(x, w[0], b[0], padding=1))
    ref = torch.relu(F.conv2d(h, w[1], b[1], padding=1) + x)
    y = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype="f64")
    np.testing.assert_allclose(y[:, :, 0], ref.numpy(), rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- P7 shift equivariance
def test_p7_shift_equivariance():
    x = rng.standard_normal((1, 3, 16, 16))
    w = rng.standard_normal((2, 3, 3, 3))
    y = oracle.conv(x, w, pad=(1, 1))
    ys = oracle.conv(np.roll(x, (2, 3), axis=(2, 3)), w, pad=(1, 1))
    np.testing.assert_allclose(ys[..., 4:-1, 5:-1], np.roll(y, (2, 3), axis=(2, 3))[..., 4:-1, 5:-1],
                               rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- bf16 rounding vs torch's cast
def test_bf16_round_matches_torch_cast():
    v = rng.standard_normal(200000).astype(np.float32) * np.float32(3.0)
    # add exact ties: bf16 value + half an ulp (representable in fp32)
    b = torch.from_numpy(v[:1000]).to(torch.bfloat16).float().numpy()
    ulp = np.abs(b) * 2.0 ** -7
    ties = (b + 0.5 * np.float32(2.0) ** np.floor(np.log2(np.abs(b) + 1e-30)) * 2.0 ** -7).astype(np.float32)
    allv = np.concatenate([v, ties, np.array([0.0, -0.0, 1.0, -1.5, 65504.0], np.float32)])
    ref = torch.from_numpy(allv).to(torch.bfloat16).double().numpy()
    got = oracle.round_bf16(allv.astype(np.float64))
    np.testing.assert_array_equal(got, ref)
    assert ulp.shape == b.shape


def test_epilogue_order_bias_residual_relu_round():
    y = np.array([1.0, -2.0, 0.3, 1.00390625 + 2 ** -9])
    r = np.array([-0.5, 1.0, -0.4, 0.0])
    oracle.epilogue(y, r, relu=True, round_mode=1)
    np.testing.assert_array_equal(y, [0.5, 0.0, 0.0, 1.0078125])


# ---------------------------------------------------------------- brick layout definition
@pytest.mark.parametrize("shape,brick,cp", [
    ((1, 8, 1, 32, 32), (1, 1, 8, 8), 8),
    ((2, 3, 1, 7, 9), (1, 1, 4, 4), 8),        # non-multiples, padded channels
    ((3, 5, 1, 56, 56), (2, 1, 16, 16), 8),    # batch blocking, 56/16 ragged
    ((1, 4, 6, 7, 5), (1, 4, 4, 4), 4),        # 3D ragged
])
def test_layout_roundtrip_and_zero_mask(shape, brick, cp):
    x = rng.standard_normal(shape)
    b = oracle.brickify(x, brick, cp)
    N, C, D, H, W = shape
    Bn, Bd, Bh, Bw = brick
    grid = [-(-N // Bn), -(-D // Bd), -(-H // Bh), -(-W // Bw)]
    assert b.size == np.prod(grid) * Bn * Bd * Bh * Bw * cp
    np.testing.assert_array_equal(oracle.unbrickify(b, shape, brick, cp), x)
    # masked positions and padded channels are zero; exactly N*C*D*H*W non-zero slots
    assert np.count_nonzero(b) == np.count_nonzero(x)
    # one element by hand: (n,c,d,h,w) -> brick ((n/Bn,d/Bd,h/Bh,w/Bw)), inner (n%Bn,..)*cp + c
    n, c, d, h, w = N - 1, C - 1, D - 1, H - 1, W - 1
    lb = ((n // Bn * grid[1] + d // Bd) * grid[2] + h // Bh) * grid[3] + w // Bw
    inner = ((((n % Bn) * Bd + d % Bd) * Bh + h % Bh) * Bw + w % Bw) * cp + c
    assert b[lb * Bn * Bd * Bh * Bw * cp + inner] == x[n, c, d, h, w]


def test_layout_brickmap_permutation():
    shape, brick, cp = (1, 2, 1, 16, 16), (1, 1, 4, 4), 4
    x = rng.standard_normal(shape)
    g = json.load(open(os.path.join(GOLDEN, "fig6_brickinfo.json")))
    bm = np.array(g["brickmap"], dtype=np.int32).reshape(-1)
    b = oracle.brickify(x, brick, cp, brickmap=bm)
    np.testing.assert_array_equal(oracle.unbrickify(b, shape, brick, cp, brickmap=bm), x)
    # Fig 6a: physical brick 0 holds logical brick (1,1) = rows 4..7, cols 4..7
    be = 16 * cp
    blk = b[:be].reshape(4, 4, cp)
    np.testing.assert_array_equal(blk[:, :, 0], x[0, 0, 0, 4:8, 4:8])


def test_fig6_brickinfo_golden():
    g = json.load(open(os.path.join(GOLDEN, "fig6_brickinfo.json")))
    bm = np.array(g["brickmap"], dtype=np.int32)
    adj = oracle.brickinfo(2, (1, 4, 4), bm.reshape(-1))
    assert adj[0].tolist() == g["eta_phys0"]
    # every in-grid neighbour relation is symmetric
    dirs = list(zip(g["di"], g["dj"]))
    for p in range(16):
        for k, (di, dj) in enumerate(dirs):
            q = adj[p, k]
            if q >= 0:
                assert adj[q, dirs.index((-di, -dj))] == p


def test_workload_recipe_is_seeded_and_bf16_representable():
    a = workloads.make_workload("cfg2", N=1, H=8, W=8)
    b = workloads.make_workload("cfg2", N=1, H=8, W=8)
    assert torch.equal(a["x"], b["x"]) and torch.equal(a["weights"][1], b["weights"][1])
    assert torch.equal(a["x"], a["x"].to(torch.bfloat16).float())
    assert torch.equal(a["weights"][0], a["weights"][0].to(torch.bfloat16).float())
    L = workloads.make_layers("cfg4")
    assert sum(l["kind"] == "conv" for l in L) == 53
    assert sum(l["kind"] == "maxpool" for l in workloads.make_layers("cfg3")) == 5


# ---------------------------------------------------------------- P6 on the branched (DAG) path
def _resnet50_prefix_torch(x, w, b):
    """ResNet-50 v1.5 prefix written out by hand with torch fp64 (no layer indices involved): stem
    conv7x7/2 + ReLU, maxpool 3x3/2 p1, conv2_x block 1 (projection shortcut), conv2_x blocks 2 and 3
    (identity shortcuts), conv3_x block 1 (stride 2 on the 3x3 and on the projection).  Epilogue
    order bias -> residual add -> ReLU.  w/b are consumed in the listed order."""
    F = torch.nn.functional
    it = iter(zip(w, b))

    def conv(h, s=1, p=0, relu=True):
        wi, bi = next(it)
        y = F.conv2d(h, wi, bi, stride=s, padding=p)
        return torch.relu(y) if relu else y

    h = conv(x, s=2, p=3)
    next(it)                                   # the pool has no weights
    h = F.max_pool2d(h, 3, 2, 1)
    for stage_stride, nblocks in ((1, 3), (2, 1)):
        for blk in range(nblocks):
            s = stage_stride if blk == 0 else 1
            a = conv(h)
            a = conv(a, s=s, p=1)
            if blk == 0:
                proj = conv(h, s=s, relu=False)
                wi, bi = next(it)
                h = torch.relu(F.conv2d(a, wi, bi) + proj)
            else:
                wi, bi = next(it)
                h = torch.relu(F.conv2d(a, wi, bi) + h)
    return h


def test_p6_dag_resnet50_prefix_vs_torch():
    """Pins run_graph's branch semantics (a layer reading a non-previous layer; a residual taken from
    a layer OUTPUT, the projection) and make_layers('cfg4')'s input/residual indices: the first 16
    layers of the cfg4 graph against the hand-written torch fp64 forward (§4.3 ResNet-50,
    L1130-1165; merged execution reproduces exactly this layer-by-layer result, L363-365)."""
    layers = workloads.make_layers("cfg4")[:16]
    assert [l["kind"] for l in layers].count("maxpool") == 1
    wl = workloads.make_graph_workload(layers, 2, 3, 1, 40, 36, 2, (1, 1, 8, 8), "f64", seed=41)
    y = oracle.run_graph(wl["layers"], wl["x"].numpy(), wl["weights"], wl["biases"], dtype="f64")
    ws = [t.double()[:, :, 0] for t in wl["weights"] if t is not None]
    bs = [t.double() for t in wl["biases"] if t is not None]
    ws.insert(1, None)
    bs.insert(1, None)
    ref = _resnet50_prefix_torch(wl["x"].double()[:, :, 0], ws, bs)
    assert y.shape[1:] == (512, 1, 5, 5)
    np.testing.assert_allclose(y[:, :, 0], ref.numpy(), rtol=1e-12, atol=1e-12)
    # the pin discriminates: block 2 adding the projection output (layer 4) instead of block 1's output
    # (layer 5) -- same shape, wrong index -- must fail it
    assert wl["layers"][8]["residual"] == 5 and wl["layers"][5]["residual"] == 4
    bad = [dict(l) for l in wl["layers"]]
    bad[8]["residual"] = 4
    with pytest.raises(AssertionError):
        yb = oracle.run_graph(bad, wl["x"].numpy(), wl["weights"], wl["biases"], dtype="f64")
        np.testing.assert_allclose(yb[:, :, 0], ref.numpy(), rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- dilated and grouped convolution (N2)
@pytest.mark.parametrize("dil,groups,s,p", [(2, 1, 1, 2), (3, 1, 1, 0), (1, 4, 1, 1), (2, 4, 2, 2), (1, 8, 1, 1)])
def test_p6_torch_conv2d_dilated_grouped(dil, groups, s, p):
    """Dilated / grouped / depthwise convs (the mergeable set beyond dense convs, L378-385) against torch fp64."""
    x = rng.standard_normal((2, 8, 13, 11))
    w = rng.standard_normal((8, 8 // groups, 3, 3))
    b = rng.standard_normal(8)
    y = oracle.conv(x, w, bias=b, stride=(s, s), pad=(p, p), dil=(dil, dil), groups=groups)
    ref = torch.nn.functional.conv2d(torch.from_numpy(x), torch.from_numpy(w), torch.from_numpy(b), stride=s,
                                     padding=p, dilation=dil, groups=groups).numpy()
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


def test_p1_delta_input_dilated():
    """Delta input: a dilated kernel's taps land d apart: y[oh, ow] = w[r, s] where oh - p + d*r = h0."""
    x = np.zeros((1, 1, 9, 9))
    x[0, 0, 4, 4] = 1.0
    w = rng.standard_normal((1, 1, 3, 3))
    y = oracle.conv(x, w, pad=(2, 2), dil=(2, 2))
    expect = np.zeros_like(y)
    for r in range(3):
        for c in range(3):
            expect[0, 0, 4 + 2 - 2 * r, 4 + 2 - 2 * c] = w[0, 0, r, c]
    np.testing.assert_array_equal(y, expect)


def test_depthwise_is_per_channel():
    """groups = C: each output channel is the 1-channel conv of its own input channel (brute force per channel)."""
    x = rng.standard_normal((1, 3, 7, 6))
    w = rng.standard_normal((3, 1, 3, 3))
    y = oracle.conv(x, w, pad=(1, 1), groups=3)
    for c in range(3):
        np.testing.assert_array_equal(y[:, c:c + 1], oracle.conv(x[:, c:c + 1], w[c:c + 1], pad=(1, 1)))


# ---------------------------------------------------------------- transposed convolution (N2)
@pytest.mark.parametrize("k,s,p,d", [(4, 2, 1, 1), (2, 2, 0, 1), (3, 2, 1, 1), (3, 1, 1, 1), (3, 1, 2, 2), (5, 3, 2, 1)])
def test_p6_torch_conv_transpose2d(k, s, p, d):
    """Transposed conv against torch fp64 (torch's weight is [Ci, Co, k]: ours, w[co, ci], transposed)."""
    x = rng.standard_normal((2, 6, 7, 9))
    w = rng.standard_normal((5, 6, k, k))
    b = rng.standard_normal(5)
    y = oracle.conv_transpose(x, w, bias=b, stride=(s, s), pad=(p, p), dil=(d, d))
    ref = torch.nn.functional.conv_transpose2d(torch.from_numpy(x), torch.from_numpy(w).transpose(0, 1).contiguous(),
                                               torch.from_numpy(b), stride=s, padding=p, dilation=d).numpy()
    assert y.shape == ref.shape
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


def test_p6_torch_conv_transpose3d():
    x = rng.standard_normal((1, 3, 4, 5, 6))
    w = rng.standard_normal((4, 3, 4, 4, 4))
    y = oracle.conv_transpose(x, w, stride=(2, 2, 2), pad=(1, 1, 1))
    ref = torch.nn.functional.conv_transpose3d(torch.from_numpy(x), torch.from_numpy(w).transpose(0, 1).contiguous(),
                                               stride=2, padding=1).numpy()
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("k,s,p,d", [(3, 2, 1, 1), (4, 2, 1, 1), (3, 1, 2, 2), (5, 3, 1, 1)])
def test_conv_transpose_is_the_adjoint(k, s, p, d):
    """The defining identity, independent of any library: <conv(x; w), y> = <x, conv_transpose(y; w^T)> with
    w^T[ci, co] = w[co, ci], whenever the transposed extent returns to the conv's input extent."""
    I = s * 7 + d * (k - 1) + 1 - 2 * p        # (I + 2p - d(k-1) - 1) divisible by s
    x = rng.standard_normal((1, 3, I, I))
    w = rng.standard_normal((4, 3, k, k))
    yc = oracle.conv(x, w, stride=(s, s), pad=(p, p), dil=(d, d))
    y = rng.standard_normal(yc.shape)
    xt = oracle.conv_transpose(y, np.ascontiguousarray(w.transpose(1, 0, 2, 3)), stride=(s, s), pad=(p, p), dil=(d, d))
    assert xt.shape == x.shape
    lhs, rhs = float(np.sum(yc * y)), float(np.sum(x * xt))
    assert abs(lhs - rhs) <= 1e-10 * max(1.0, abs(lhs))


def test_p1_delta_input_transposed():
    """Delta input: one input element at i spreads the kernel to outputs s*i - p + d*t."""
    x = np.zeros((1, 1, 5, 5))
    x[0, 0, 2, 3] = 1.0
    w = rng.standard_normal((2, 1, 4, 4))
    y = oracle.conv_transpose(x, w, stride=(2, 2), pad=(1, 1))
    expect = np.zeros_like(y)
    for r in range(4):
        for c in range(4):
            oh, ow = 2 * 2 - 1 + r, 2 * 3 - 1 + c
            if 0 <= oh < y.shape[2] and 0 <= ow < y.shape[3]:
                expect[0, :, oh, ow] = w[:, 0, r, c]
    np.testing.assert_array_equal(y, expect)
