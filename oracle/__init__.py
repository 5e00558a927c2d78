"""BrickDL CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference` legs may
import this package.  The product path (paper_conf_icpp_lakshminarasimhan24_b200) never does;
the two share no code (only the seeded generators in
paper_conf_icpp_lakshminarasimhan24_b200/workloads.py, which hold no arithmetic of the method).

Python side of the oracle: a ctypes shim over oracle.c (fp64 direct convolution, max-pool,
epilogue, bf16 rounding, brick layout definition, BrickInfo) plus `run_graph`, the plain
layer-by-layer evaluation of a layer graph in the order it is listed -- which is what merged
execution must reproduce, since it only reorders work.
Every function cites its passage in oracle.c's header.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

_dp = ctypes.POINTER(ctypes.c_double)
_ip = ctypes.POINTER(ctypes.c_int32)
_i = ctypes.c_int


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (plain C, -O2, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c99",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            L.oracle_round_bf16.restype = ctypes.c_double
            L.oracle_round_bf16.argtypes = [ctypes.c_double]
            L.oracle_conv.restype = None
            L.oracle_conv.argtypes = [_dp, _i, _i, _i, _i, _i, _dp, _dp, _i] + [_i] * 12 + [_dp, _i, _i, _i]
            L.oracle_conv_transpose.restype = None
            L.oracle_conv_transpose.argtypes = [_dp, _i, _i, _i, _i, _i, _dp, _dp, _i] + [_i] * 12 + [_dp, _i, _i, _i]
            L.oracle_maxpool.restype = None
            L.oracle_maxpool.argtypes = [_dp, _i, _i, _i, _i, _i] + [_i] * 9 + [_dp, _i, _i, _i]
            L.oracle_epilogue.restype = None
            L.oracle_epilogue.argtypes = [_dp, _dp, ctypes.c_size_t, _i, _i]
            L.oracle_brickify.restype = None
            L.oracle_brickify.argtypes = [_dp] + [_i] * 10 + [_ip, _dp]
            L.oracle_unbrickify.restype = None
            L.oracle_unbrickify.argtypes = [_dp] + [_i] * 10 + [_ip, _dp]
            L.oracle_brickinfo.restype = None
            L.oracle_brickinfo.argtypes = [_i, _i, _i, _i, _ip, _ip]
            _lib = L
    return _lib


def _d(a: np.ndarray):
    assert a.dtype == np.float64 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(_dp)


def _as5(x):
    x = np.ascontiguousarray(np.asarray(x, dtype=np.float64))
    if x.ndim == 4:
        x = x[:, :, None]
    return np.ascontiguousarray(x)


def set_threads(n: int) -> None:
    os.environ["OMP_NUM_THREADS"] = str(n)


def round_bf16(x):
    """Elementwise bf16 round-to-nearest-even (oracle.c: oracle_round_bf16)."""
    L = lib()
    a = np.ascontiguousarray(np.asarray(x, dtype=np.float64)).copy()
    flat = a.reshape(-1)
    L.oracle_epilogue(_d(flat), None, flat.size, 0, 1)
    return a


def conv(x, w, bias=None, stride=(1, 1, 1), pad=(0, 0, 0), dil=(1, 1, 1), groups=1):
    """Direct convolution (cross-correlation), fp64.  x [N,Ci,D,H,W] (or 4-D), w [Co,Ci/groups,kd,kh,kw].
    groups > 1 (grouped / depthwise conv): by definition, output channels [g*Co/G, (g+1)*Co/G) are the conv of
    input channels [g*Ci/G, (g+1)*Ci/G) alone -- G independent oracle_conv calls on the channel slices."""
    if groups > 1:
        xa, wa = np.asarray(x, dtype=np.float64), np.asarray(w, dtype=np.float64)
        ci, co = xa.shape[1] // groups, wa.shape[0] // groups
        ys = [conv(xa[:, g * ci:(g + 1) * ci], wa[g * co:(g + 1) * co],
                   None if bias is None else np.asarray(bias, np.float64)[g * co:(g + 1) * co], stride, pad, dil)
              for g in range(groups)]
        return np.ascontiguousarray(np.concatenate(ys, axis=1))
    four = np.asarray(x).ndim == 4
    x = _as5(x)
    w = np.asarray(w, dtype=np.float64)
    if w.ndim == 4:
        w = w[:, :, None]
    w = np.ascontiguousarray(w)
    N, Ci, D, H, W = x.shape
    Co, Ci2, kd, kh, kw = w.shape
    assert Ci == Ci2
    if four:
        stride, pad, dil = (1,) + tuple(stride[-2:]), (0,) + tuple(pad[-2:]), (1,) + tuple(dil[-2:])
    Do = (D + 2 * pad[0] - dil[0] * (kd - 1) - 1) // stride[0] + 1
    Ho = (H + 2 * pad[1] - dil[1] * (kh - 1) - 1) // stride[1] + 1
    Wo = (W + 2 * pad[2] - dil[2] * (kw - 1) - 1) // stride[2] + 1
    y = np.empty((N, Co, Do, Ho, Wo), dtype=np.float64)
    b = None if bias is None else np.ascontiguousarray(np.asarray(bias, dtype=np.float64))
    lib().oracle_conv(_d(x), N, Ci, D, H, W, _d(w), None if b is None else _d(b), Co,
                      kd, kh, kw, *stride, *pad, *dil, _d(y), Do, Ho, Wo)
    return y[:, :, 0] if four else y


def conv_transpose(x, w, bias=None, stride=(1, 1, 1), pad=(0, 0, 0), dil=(1, 1, 1)):
    """Transposed convolution, fp64 (oracle_conv_transpose: every input element scattered through the kernel).
    x [N,Ci,D,H,W] (or 4-D), w [Co,Ci,kd,kh,kw]: w[co,ci,t] carries input channel ci to output channel co.
    Output extent (I-1)s - 2p + d(k-1) + 1."""
    four = np.asarray(x).ndim == 4
    x = _as5(x)
    w = np.asarray(w, dtype=np.float64)
    if w.ndim == 4:
        w = w[:, :, None]
    w = np.ascontiguousarray(w)
    N, Ci, D, H, W = x.shape
    Co, Ci2, kd, kh, kw = w.shape
    assert Ci == Ci2
    if four:
        stride, pad, dil = (1,) + tuple(stride[-2:]), (0,) + tuple(pad[-2:]), (1,) + tuple(dil[-2:])
    Do = (D - 1) * stride[0] - 2 * pad[0] + dil[0] * (kd - 1) + 1
    Ho = (H - 1) * stride[1] - 2 * pad[1] + dil[1] * (kh - 1) + 1
    Wo = (W - 1) * stride[2] - 2 * pad[2] + dil[2] * (kw - 1) + 1
    y = np.empty((N, Co, Do, Ho, Wo), dtype=np.float64)
    b = None if bias is None else np.ascontiguousarray(np.asarray(bias, dtype=np.float64))
    lib().oracle_conv_transpose(_d(x), N, Ci, D, H, W, _d(w), None if b is None else _d(b), Co,
                                kd, kh, kw, *stride, *pad, *dil, _d(y), Do, Ho, Wo)
    return y[:, :, 0] if four else y


def maxpool(x, k, stride, pad):
    """Max pooling, out-of-range positions ignored.  k/stride/pad are 3-tuples (d,h,w)."""
    four = np.asarray(x).ndim == 4
    x = _as5(x)
    N, C, D, H, W = x.shape
    if four:
        k, stride, pad = (1,) + tuple(k[-2:]), (1,) + tuple(stride[-2:]), (0,) + tuple(pad[-2:])
    Do = (D + 2 * pad[0] - k[0]) // stride[0] + 1
    Ho = (H + 2 * pad[1] - k[1]) // stride[1] + 1
    Wo = (W + 2 * pad[2] - k[2]) // stride[2] + 1
    y = np.empty((N, C, Do, Ho, Wo), dtype=np.float64)
    lib().oracle_maxpool(_d(x), N, C, D, H, W, *k, *stride, *pad, _d(y), Do, Ho, Wo)
    return y[:, :, 0] if four else y


def epilogue(y, residual=None, relu=False, round_mode=0):
    """In place: y += residual; ReLU; round (0 none, 1 bf16, 2 fp32).  Returns y."""
    assert y.dtype == np.float64 and y.flags["C_CONTIGUOUS"]
    r = None
    if residual is not None:
        r = np.ascontiguousarray(np.asarray(residual, dtype=np.float64))
        assert r.shape == y.shape
    lib().oracle_epilogue(_d(y), None if r is None else _d(r), y.size, int(relu), int(round_mode))
    return y


def brickify(x, brick, c_pad, brickmap=None):
    """Brick layout definition; x [N,C,D,H,W] -> flat array of nbricks*brick_elems (fp64)."""
    x = _as5(x)
    N, C, D, H, W = x.shape
    Bn, Bd, Bh, Bw = brick
    nb = (-(-N // Bn)) * (-(-D // Bd)) * (-(-H // Bh)) * (-(-W // Bw))
    out = np.empty(nb * Bn * Bd * Bh * Bw * c_pad, dtype=np.float64)
    bm = None
    if brickmap is not None:
        bm = np.ascontiguousarray(np.asarray(brickmap, dtype=np.int32))
    lib().oracle_brickify(_d(x), N, C, D, H, W, Bn, Bd, Bh, Bw, c_pad,
                          None if bm is None else bm.ctypes.data_as(_ip), _d(out))
    return out


def unbrickify(src, shape, brick, c_pad, brickmap=None):
    N, C, D, H, W = shape
    Bn, Bd, Bh, Bw = brick
    src = np.ascontiguousarray(np.asarray(src, dtype=np.float64))
    x = np.empty((N, C, D, H, W), dtype=np.float64)
    bm = None
    if brickmap is not None:
        bm = np.ascontiguousarray(np.asarray(brickmap, dtype=np.int32))
    lib().oracle_unbrickify(_d(src), N, C, D, H, W, Bn, Bd, Bh, Bw, c_pad,
                            None if bm is None else bm.ctypes.data_as(_ip), _d(x))
    return x


def brickinfo(nsp, grid, brickmap=None):
    """Adjacency [nbricks][3^nsp - 1] in physical order (Fig 6c direction order)."""
    nbd, nbh, nbw = grid
    nb = nbd * nbh * nbw
    ndir = (27 if nsp == 3 else 9) - 1
    adj = np.empty((nb, ndir), dtype=np.int32)
    bm = None
    if brickmap is not None:
        bm = np.ascontiguousarray(np.asarray(brickmap, dtype=np.int32).reshape(-1))
    lib().oracle_brickinfo(nsp, nbd, nbh, nbw, None if bm is None else bm.ctypes.data_as(_ip),
                           adj.ctypes.data_as(_ip))
    return adj


def run_graph(layers, x, weights, biases, dtype="bf16", keep_all=False):
    """Layer-by-layer evaluation of a layer graph (workloads.make_layers format), fp64 accumulation.

    Each layer: conv (+bias) or maxpool on the output of layer `input` (-1 = graph input), then
    + output of layer `residual`, ReLU, and rounding to the storage dtype (bf16 RNE / fp32),
    the epilogue order of SURVEY Q14.  Returns the last layer's output (or all outputs).
    """
    rmode = {"bf16": 1, "f32": 2, "f64": 0}[dtype]
    x = _as5(x)
    outs = []
    for l, w, b in zip(layers, weights, biases):
        src = x if l["input"] == -1 else outs[l["input"]]
        if l["kind"] == "conv" and l.get("transposed"):
            y = conv_transpose(src, np.asarray(w, dtype=np.float64), None if b is None else np.asarray(b, np.float64),
                               stride=l["stride"], pad=l["pad"], dil=l.get("dil", (1, 1, 1)))
        elif l["kind"] == "conv":
            y = conv(src, np.asarray(w, dtype=np.float64), None if b is None else np.asarray(b, np.float64),
                     stride=l["stride"], pad=l["pad"], dil=l.get("dil", (1, 1, 1)), groups=l.get("groups", 1))
        else:
            y = maxpool(src, l["k"], l["stride"], l["pad"])
        res = None
        if l["residual"] is not None:
            res = x if l["residual"] == -1 else outs[l["residual"]]
        epilogue(y, res, l["relu"], rmode)
        outs.append(y)
    return outs if keep_all else outs[-1]
