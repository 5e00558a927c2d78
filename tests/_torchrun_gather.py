"""Worker for test_torchrun_batch_gather (launched by torch.distributed.run, env:// rendezvous on 127.0.0.1): the
strong-scaling batch runner's gather on CPU tensors over gloo, checked against the unsharded computation."""
import os
import sys

import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_lakshminarasimhan24_b200 import parallel  # noqa: E402


def layer(x, out):
    w = torch.linspace(-1, 1, 4 * 3 * 3 * 3, dtype=torch.float64).reshape(4, 3, 3, 3)
    out.copy_(torch.relu(torch.nn.functional.conv2d(x[:, :, 0], w, padding=1))[:, :, None])
    return out


def main():
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    n = 3 * world
    x_all = torch.randn(n, 3, 1, 7, 6, generator=torch.Generator().manual_seed(11), dtype=torch.float64)
    run = parallel.BatchRunner(n, (4, 1, 7, 6), rank, world, micro=3, compute=layer, device="cpu", dtype=torch.float64)
    y = run.forward(x_all[run.global_images()].contiguous())
    ok = torch.equal(y, layer(x_all, torch.empty(n, 4, 1, 7, 6, dtype=torch.float64)))
    t = torch.tensor([int(ok)])
    dist.all_reduce(t, op=dist.ReduceOp.MIN)
    if rank == 0:
        print("GATHER_OK" if t.item() == 1 else "GATHER_MISMATCH")
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
