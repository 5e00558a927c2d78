"""Seeded synthetic workloads shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method: it only describes layer graphs (shapes) and draws
seeded random inputs, weights and biases.  Both `oracle/` and the product path consume what it
returns; neither imports the other.

Shapes follow the paper's workloads (§4.1-§4.5) as mapped in SURVEY.md §8(d):
  cfg1  2-layer 3x3 conv+ReLU chain, fp32, N=1 C=8 32x32, 8x8 bricks          (parity config)
  cfg2  ResNet-18 conv2_x basic block, bf16, N=64 C=64 56x56, 8x8 bricks      (bench config)
  cfg3  VGG-16 conv stack (13 convs + 5 pools), bf16, N=128 224x224
  cfg4  ResNet-50 v1.5 conv backbone, bf16, N=256 224x224
  cfg5  3D chain of 4 conv3x3x3 C=32 over 128^3, bf16, 4x4x4 bricks (Fig 10/11 analogue, L1388-1536)

Recipe: x ~ N(0,1) drawn in fp32 (seed 1000+cfg), weights He-normal
std = sqrt(2/fan_in) (seed 2000+cfg), bias ~ U(-0.1, 0.1) (seed 3000+cfg); the last conv of a
residual branch is scaled by 0.5.  For bf16 configurations x and w are rounded to bf16 (RNE, by
torch's dtype cast) *here*, so the bf16 values are the ground truth for both sides; bias stays fp32.

Layer dict keys:
  kind        "conv" | "maxpool"
  cin, cout   channels (maxpool: cin == cout)
  k, stride, pad   3-tuples over (d, h, w); 2D layers have k[0] = 1, stride[0] = 1, pad[0] = 0
  relu        bool, applied after bias (+ residual)
  input       index of the layer whose output this layer reads; -1 = graph input
  residual    None, or index of the layer whose output is added before ReLU; -1 = graph input
  wscale      multiplier folded into the synthetic weights (0.5 on residual-branch last convs)
"""
from __future__ import annotations

import math

import torch

__all__ = ["CONFIGS", "make_layers", "make_workload", "make_graph_workload", "conv", "pool", "layer_out_shape"]

CONFIGS = {
    "cfg1": dict(nsp=2, N=1, C=8, D=1, H=32, W=32, dtype="f32", brick=(1, 1, 8, 8)),
    "cfg2": dict(nsp=2, N=64, C=64, D=1, H=56, W=56, dtype="bf16", brick=(1, 1, 8, 8)),
    "cfg3": dict(nsp=2, N=128, C=3, D=1, H=224, W=224, dtype="bf16", brick=(1, 1, 8, 8)),
    "cfg4": dict(nsp=2, N=256, C=3, D=1, H=224, W=224, dtype="bf16", brick=(1, 1, 8, 8)),
    "cfg5": dict(nsp=3, N=1, C=32, D=128, H=128, W=128, dtype="bf16", brick=(1, 4, 4, 4)),
}
_CFG_NUM = {"cfg1": 1, "cfg2": 2, "cfg3": 3, "cfg4": 4, "cfg5": 5}


def _conv(cin, cout, k=3, s=1, p=None, relu=True, inp=None, res=None, wscale=1.0, nsp=2, dil=1, groups=1,
          transposed=False):
    if p is None:
        p = dil * (k - 1) // 2 if not transposed else (dil * (k - 1) + 1 - s) // 2   # transposed: output = s * input
    if nsp == 3:
        kk, ss, pp, dd = (k, k, k), (s, s, s), (p, p, p), (dil, dil, dil)
    else:
        kk, ss, pp, dd = (1, k, k), (1, s, s), (0, p, p), (1, dil, dil)
    return dict(kind="conv", cin=cin, cout=cout, k=kk, stride=ss, pad=pp, relu=relu,
                input=inp, residual=res, wscale=wscale, dil=dd, groups=groups, transposed=bool(transposed))


def _pool(c, k, s, p):
    return dict(kind="maxpool", cin=c, cout=c, k=(1, k, k), stride=(1, s, s), pad=(0, p, p),
                relu=False, input=None, residual=None, wscale=1.0)


def make_layers(cfg: str, C: int | None = None, nlayers: int | None = None):
    """Layer graph of a configuration (inputs resolved: `input` None -> previous layer)."""
    c = CONFIGS[cfg]
    C = C if C is not None else c["C"]
    L = []
    if cfg == "cfg1":
        n = nlayers or 2
        L = [_conv(C, C) for _ in range(n)]
    elif cfg == "cfg2":
        # ResNet-18 conv2_x basic block: conv-relu, conv (x0.5), + x, relu.
        L = [_conv(C, C), _conv(C, C, res=-1, wscale=0.5)]
    elif cfg == "cfg5":
        n = nlayers or 4
        L = [_conv(C, C, nsp=3) for _ in range(n)]
    elif cfg == "cfg3":
        cin = C
        for stage in ([64, 64], [128, 128], [256, 256, 256], [512, 512, 512], [512, 512, 512]):
            for w in stage:
                L.append(_conv(cin, w))
                cin = w
            L.append(_pool(cin, 2, 2, 0))
    elif cfg == "cfg4":
        L.append(_conv(C, 64, k=7, s=2, p=3))
        L.append(_pool(64, 3, 2, 1))
        cin = 64
        for width, nblocks, stride in ((64, 3, 1), (128, 4, 2), (256, 6, 2), (512, 3, 2)):
            for b in range(nblocks):
                s = stride if b == 0 else 1
                blk_in = len(L) - 1
                L.append(_conv(cin, width, k=1, inp=blk_in))
                L.append(_conv(width, width, k=3, s=s))
                if b == 0:
                    L.append(_conv(cin, width * 4, k=1, s=s, relu=False, inp=blk_in))  # projection
                    res = len(L) - 1
                    L.append(_conv(width, width * 4, k=1, inp=len(L) - 2, res=res, wscale=0.5))
                else:
                    L.append(_conv(width, width * 4, k=1, res=blk_in, wscale=0.5))
                cin = width * 4
    else:
        raise KeyError(cfg)
    for i, l in enumerate(L):
        if l["input"] is None:
            l["input"] = i - 1
    return L


def layer_out_shape(layer, D, H, W):
    """Output spatial extent of one layer: floor((I + 2p - d(k-1) - 1)/s) + 1 per dim (transposed conv:
    (I-1)s - 2p + d(k-1) + 1)."""
    out = []
    for I, k, s, p, d in zip((D, H, W), layer["k"], layer["stride"], layer["pad"], layer.get("dil", (1, 1, 1))):
        if layer.get("transposed"):
            out.append((I - 1) * s - 2 * p + d * (k - 1) + 1)
        else:
            out.append((I + 2 * p - d * (k - 1) - 1) // s + 1)
    return tuple(out)


def make_workload(cfg: str, N=None, C=None, D=None, H=None, W=None, nlayers=None, seed_offset=0,
                  input_seed_offset=0):
    """Seeded synthetic input, weights and biases for a configuration (optionally resized).

    Returns dict(cfg, nsp, dtype, N, C, D, H, W, brick, layers, x, weights, biases) where
      x        torch.float32 [N, C, D, H, W] (bf16-representable for bf16 configs)
      weights  list (per layer; None for pools) of torch.float32 [Co, Ci, kd, kh, kw]
      biases   list of torch.float32 [Co] or None
    """
    c = dict(CONFIGS[cfg])
    for k, v in dict(N=N, C=C, D=D, H=H, W=W).items():
        if v is not None:
            c[k] = v
    num = _CFG_NUM[cfg] + seed_offset
    layers = make_layers(cfg, C=c["C"], nlayers=nlayers)
    wl = make_graph_workload(layers, c["N"], c["C"], c["D"], c["H"], c["W"], c["nsp"], c["brick"], c["dtype"],
                             seed=num, input_seed_offset=input_seed_offset)
    wl["cfg"] = cfg
    return wl


def conv(cin, cout, k=3, s=1, p=None, relu=True, inp=None, res=None, wscale=1.0, nsp=2, dil=1, groups=1,
         transposed=False):
    """Layer dict of a conv (public form of the graph builder used by the configurations).  dil: dilation;
    groups: grouped conv (groups = cin: depthwise), weights [cout, cin/groups, k...]; transposed: transposed conv
    (weights [cout, cin, k...], w[co, ci] carrying ci to co; default padding makes the output s x the input)."""
    return _conv(cin, cout, k, s, p, relu, inp, res, wscale, nsp, dil, groups, transposed)


def pool(c, k, s, p):
    return _pool(c, k, s, p)


def make_graph_workload(layers, N, C, D, H, W, nsp, brick, dtype, seed=0, input_seed_offset=0):
    """Seeded synthetic input, weights and biases for an arbitrary layer graph (same recipe as the
    configurations: seeds 1000/2000/3000 + seed)."""
    layers = [dict(l) for l in layers]
    for i, l in enumerate(layers):
        if l["input"] is None:
            l["input"] = i - 1
    bf16 = dtype == "bf16"
    g = torch.Generator().manual_seed(1000 + seed + 100 * input_seed_offset)  # per-shard inputs (ranks)
    x = torch.randn(N, C, D, H, W, generator=g, dtype=torch.float32)
    if bf16:
        x = x.to(torch.bfloat16).to(torch.float32)
    gw = torch.Generator().manual_seed(2000 + seed)
    gb = torch.Generator().manual_seed(3000 + seed)
    weights, biases = [], []
    for l in layers:
        if l["kind"] != "conv":
            weights.append(None)
            biases.append(None)
            continue
        kd, kh, kw = l["k"]
        cin_g = l["cin"] // l.get("groups", 1)
        fan_in = cin_g * kd * kh * kw
        w = torch.randn(l["cout"], cin_g, kd, kh, kw, generator=gw, dtype=torch.float32)
        w = w * (math.sqrt(2.0 / fan_in) * l["wscale"])
        if bf16:
            w = w.to(torch.bfloat16).to(torch.float32)
        b = (torch.rand(l["cout"], generator=gb, dtype=torch.float32) * 0.2 - 0.1)
        weights.append(w)
        biases.append(b)
    return dict(cfg="custom", nsp=nsp, dtype=dtype, N=N, C=C, D=D, H=H, W=W, brick=tuple(brick), layers=layers,
                x=x, weights=weights, biases=biases)
