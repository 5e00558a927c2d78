"""The generic kernel's alternative code paths produce the same bits as the paths they replace.

Several choices of `chain_tc_gen.cu` are made per subgraph at launch time, each with an A/B switch read once per
process from the environment: the epilogue warp count (BDL_GEN_EPIW: 8 or 12, a template instantiation), the TMA box
per brick row of the 1x1 layers (BDL_GEN_TMA4=0: one box per pixel row), the element-strided TMA rows of 3x3
stride-2 layers (BDL_GEN_TMA3=0: cp.async), the shallow-K weight-stage split (BDL_GEN_NW2), and the epilogue's
bias source (BDL_GEN_BIAS_SMEM=0: a global load + shuffles per item instead of the shared fp32 table).  Loads and the
epilogue's partition of work never change an output element's accumulation order, so every setting must give
bit-identical outputs.  Each setting runs in its own process (the switches are static) on a reduced ResNet-50
(stem, pools, projection and identity bottlenecks, stride-2 3x3 convs, 1x1 layers at brick-misaligned extents) and
a reduced VGG-16 (no residuals: the 8-warp epilogue by default).
"""
import hashlib
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import hashlib, sys
sys.path.insert(0, sys.argv[1])
import torch
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads
cfg, N, H = sys.argv[2], int(sys.argv[3]), int(sys.argv[4])
wl = workloads.make_workload(cfg, N=N, H=H, W=H)
plan = engine.plan_from_workload(wl)
y = plan.forward(wl["x"]).contiguous().view(torch.int16).cpu().numpy()
print(hashlib.sha256(y.tobytes()).hexdigest())
"""


def digest(cfg, N, H, **env):
    e = dict(os.environ)
    e.update({k: str(v) for k, v in env.items()})
    r = subprocess.run([sys.executable, "-c", SCRIPT, ROOT, cfg, str(N), str(H)], env=e, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    return r.stdout.strip().splitlines()[-1]


@pytest.mark.parametrize("cfg,N,H", [("cfg4", 3, 120), ("cfg3", 2, 88)])
def test_alternative_paths_bit_identical(cfg, N, H):
    base = digest(cfg, N, H)
    for env in (dict(BDL_GEN_EPIW=8), dict(BDL_GEN_EPIW=12), dict(BDL_GEN_TMA4=0), dict(BDL_GEN_TMA3=0),
                dict(BDL_GEN_NW2=0), dict(BDL_GEN_NW2=1), dict(BDL_GEN_BIAS_SMEM=0)):
        assert digest(cfg, N, H, **env) == base, env
