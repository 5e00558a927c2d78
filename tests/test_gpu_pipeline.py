"""The serving path (engine.HostPipeline): pipelined host-to-host inference must return, for every request,
exactly what plan.forward returns for it (same kernels, same per-output K order), whatever the overlap of
H2D, compute and D2H across requests; and the oracle bound holds."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_icpp_lakshminarasimhan24_b200 import engine, workloads

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("slots", [2, 3])
def test_host_pipeline_matches_forward(slots):
    wls = [workloads.make_workload("cfg2", N=2, H=20, W=20, input_seed_offset=i) for i in range(5)]
    plan = engine.plan_from_workload(wls[0])
    xs = [w["x"].to(plan.tdtype).contiguous().pin_memory() for w in wls]
    pipe = engine.HostPipeline(plan, slots=slots)
    outs = pipe.run(xs)
    assert len(outs) == len(xs)
    for w, x, y in zip(wls, xs, outs):
        ref = plan.forward(x.cuda()).cpu()
        assert torch.equal(y, ref)
    o = oracle.run_graph(wls[3]["layers"], wls[3]["x"].numpy(), wls[3]["weights"], wls[3]["biases"], dtype="bf16")
    err = float(np.max(np.abs(outs[3].float().numpy() - o)) / np.max(np.abs(o)))
    assert err <= 2e-2, err


def test_host_pipeline_callback_order():
    wl = workloads.make_workload("cfg1")
    plan = engine.plan_from_workload(wl)
    xs = [(wl["x"] * (1 + i)).contiguous().pin_memory() for i in range(4)]
    seen = []
    engine.HostPipeline(plan).run(xs, on_output=lambda k, y: seen.append((k, y.clone())))
    assert [k for k, _ in seen] == [0, 1, 2, 3]
    for (k, y), x in zip(seen, xs):
        assert torch.equal(y, plan.forward(x.cuda()).cpu())
