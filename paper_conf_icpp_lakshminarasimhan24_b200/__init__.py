"""B200-native BrickDL merged conv-chain engine -- Python binding of the C ABI (include/brickdl.h).

This module only marshals arguments: every step of the path (brickify, merged subgraphs,
unbrickify, weight packing) runs in the CUDA kernels of libbrickdl.so.  The library is loaded
lazily; if it is missing, every entry point raises (there is no fallback implementation).
PyTorch is used by `engine.py` for device memory and streams only.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libbrickdl.so")

BDL_OK, BDL_EINVAL, BDL_EUNSUPPORTED, BDL_ENOMEM, BDL_ECUDA, BDL_EDEADLOCK = range(6)
BDL_F32, BDL_BF16 = 0, 1
BDL_MODE_AUTO, BDL_MODE_PADDED, BDL_MODE_MEMOIZED, BDL_MODE_UNMERGED = range(4)
BDL_OP_CONV, BDL_OP_MAXPOOL = 0, 1
BDL_NO_RESIDUAL, BDL_GRAPH_INPUT = -2, -1
MODE_NAMES = {1: "padded", 2: "memoized", 3: "unmerged"}
KERNEL_NAMES = {0: "cuda-core brick", 1: "tcgen05 band", 2: "tcgen05 generic"}

_i32, _i64, _f64, _vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_double, ctypes.c_void_p


class bdl_layout(ctypes.Structure):
    _fields_ = [("nsp", _i32), ("dtype", _i32), ("N", _i64), ("C", _i64), ("D", _i64), ("H", _i64),
                ("W", _i64), ("Bn", _i32), ("Bd", _i32), ("Bh", _i32), ("Bw", _i32), ("c_pad", _i32),
                ("elem_bytes", _i32), ("nb", _i64 * 4), ("nbricks", _i64), ("brick_elems", _i64),
                ("brick_bytes", _i64), ("total_bytes", _i64), ("brickmap", _vp)]


class bdl_layer(ctypes.Structure):
    _fields_ = [("kind", _i32), ("cin", _i32), ("cout", _i32), ("k", _i32 * 3), ("stride", _i32 * 3),
                ("pad", _i32 * 3), ("relu", _i32), ("input", _i32), ("residual", _i32), ("w", _vp),
                ("bias", _vp), ("dil", _i32 * 3), ("groups", _i32), ("transposed", _i32)]


class bdl_plan_opts(ctypes.Structure):
    _fields_ = [("delta_threshold", _f64), ("tau", _i64), ("bcand", _i32 * 4), ("onchip_budget", _i64),
                ("force_mode", _i32), ("force_brick", _i32), ("max_subgraph_layers", _i32),
                ("num_sms", _i32), ("schedule_seed", _i32), ("memo_defer", _i32), ("group_waves", _i32),
                ("fuse_pool", _i32)]


class BrickDLError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"brickdl status {status}: {msg}")
        self.status = status


_P = ctypes.POINTER
_SIGS = {
    "bdl_plan_opts_default": (None, [_P(bdl_plan_opts)]),
    "bdl_layout_init": (_i32, [_P(bdl_layout), _i32, _i64, _i64, _i64, _i64, _i64, _i32, _i32, _i32, _i32, _i32]),
    "bdl_brickinfo": (_i32, [_P(bdl_layout), _vp, _vp]),
    "bdl_brickify": (_i32, [_P(bdl_layout), _vp, _vp, _vp]),
    "bdl_unbrickify": (_i32, [_P(bdl_layout), _vp, _vp, _vp]),
    "bdl_graph_partition": (_i32, [_P(bdl_layer), _i32, _P(bdl_layout), _P(bdl_plan_opts), _P(_vp)]),
    "bdl_plan_num_subgraphs": (_i32, [_vp]),
    "bdl_plan_subgraph": (_i32, [_vp, _i32, _P(_i32), _P(_i32), _P(_i32), _P(_i32), _P(_f64), _P(_i32)]),
    "bdl_plan_set_mode": (_i32, [_vp, _i32, _i32]),
    "bdl_plan_out_layout": (_i32, [_vp, _P(bdl_layout)]),
    "bdl_plan_workspace_bytes": (_i64, [_vp]),
    "bdl_plan_prepare": (_i32, [_vp, _vp, _vp]),
    "bdl_run_subgraph": (_i32, [_vp, _i32, _vp, _vp, _vp, _vp]),
    "bdl_run": (_i32, [_vp, _vp, _vp, _vp, _vp]),
    "bdl_run_dense": (_i32, [_vp, _vp, _vp, _vp, _vp]),
    "bdl_plan_launches_per_run": (_i32, [_vp]),
    "bdl_plan_counters": (_i32, [_vp, _i32, _vp, _vp, _P(ctypes.c_uint64)]),
    "bdl_plan_destroy": (None, [_vp]),
    "bdl_last_error": (ctypes.c_char_p, []),
    "bdl_version": (ctypes.c_char_p, []),
    "bdl_plan_subgraph_model": (_i32, [_vp, _i32, _P(_f64), _P(_i64), _P(_i32), _P(_i32)]),
    "bdl_plan_subgraph_cta_pair": (_i32, [_vp, _i32]),
    "bdl_region_extents": (_i32, [_P(bdl_layer), _i32, _i32, _i32, _i32, _P(_i64)]),
    "bdl_model_brick": (_i32, [_P(bdl_plan_opts), _i32, _i64, _i64, _i64, _i64, _P(_i64)]),
}
EXPORTS = tuple(_SIGS)

_lib = None


def lib():
    """Load libbrickdl.so (raises if it has not been built: no fallback path exists)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build() "
                               "(python -m paper_conf_icpp_lakshminarasimhan24_b200.build)")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(status):
    if status != BDL_OK:
        raise BrickDLError(status, lib().bdl_last_error().decode())
    return status


def _wrap(name):
    def f(*args):
        return getattr(lib(), name)(*args)
    f.__name__ = name
    return f


# same names as the C ABI (argument marshalling only)
for _n in EXPORTS:
    globals()[_n] = _wrap(_n)

__all__ = ["lib", "check", "bdl_layout", "bdl_layer", "bdl_plan_opts", "BrickDLError", *EXPORTS]
