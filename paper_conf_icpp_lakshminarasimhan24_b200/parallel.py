"""Multi-GPU plumbing: one process per GPU.

Merged execution never crosses images (bricks block the batch only within a brick, PAPER.md
L374-376, L738-739), so an inference batch shards trivially across ranks: each rank runs the whole
merged plan on its share of the images.  Two ways to use that:
  * weak scaling (bench.py default): every rank runs its own batch; no data-path collective;
  * strong scaling (BatchRunner): a fixed global batch is split over the ranks in
    micro-batches and the outputs are all-gathered (NCCL over NVLink) on a communication stream while the
    next micro-batch computes -- the only data-path collective the north_star allows ("NCCL over NVLink is
    used only to gather outputs").
"""
from __future__ import annotations

import os


def shard(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous image range [lo, hi) of `rank`; sizes differ by at most one image."""
    if world <= 0 or not (0 <= rank < world):
        raise ValueError("bad rank/world")
    base, extra = divmod(n_total, world)
    lo = rank * base + min(rank, extra)
    hi = lo + base + (1 if rank < extra else 0)
    return lo, hi


def micro_batches(n_total: int, world: int, micro: int):
    """Global image ranges of the strong-scaling schedule: micro-batch i of rank r holds images
    [(i*world + r)*mb, (i*world + r + 1)*mb) with mb = n_total / (world*micro).  All-gathering micro-batch i
    over the ranks (rank-major) then yields the contiguous global images [i*world*mb, (i+1)*world*mb), so each
    gather lands directly in its final place in the output batch.  Returns mb and, per rank, the list of ranges."""
    if world <= 0 or micro <= 0 or n_total % (world * micro):
        raise ValueError(f"batch {n_total} must split into {world} ranks x {micro} micro-batches")
    mb = n_total // (world * micro)
    return mb, [[((i * world + r) * mb, (i * world + r + 1) * mb) for i in range(micro)] for r in range(world)]


class BatchRunner:
    """Strong scaling over the batch with an overlapped output gather (one rank's share).

    forward(x_local) takes this rank's micro-batches stacked as [micro*mb, C, D, H, W] (images in the order of
    micro_batches()[rank]), computes micro-batch i with `compute(x_i, out=y_i)` on the current stream and
    all-gathers y_i into the output batch on a communication stream (torch.distributed all_gather_into_tensor:
    NCCL over NVLink/NVSwitch on GPUs, gloo on CPU) while micro-batch i+1 computes.  The result is the whole
    global batch [n_total, ...] on every rank, in global image order.  gather=False leaves the outputs sharded
    (the paper's per-GPU runs).  `compute` defaults to a merged-execution Plan of mb images.
    """

    def __init__(self, n_total, out_shape, rank, world, micro=2, compute=None, plan=None, device="cuda", dtype=None,
                 group=None):
        import torch
        self.mb, ranges = micro_batches(n_total, world, micro)
        self.ranges = ranges[rank]
        self.rank, self.world, self.micro, self.group = rank, world, micro, group
        self.plan = plan
        if compute is None:
            if plan is None:
                raise ValueError("BatchRunner needs a plan or a compute function")
            compute = lambda x, out: plan.forward_into(x, out)   # noqa: E731
        self.compute = compute
        dtype = dtype if dtype is not None else (plan.tdtype if plan is not None else torch.float32)
        self.device = torch.device(device)
        self.y_local = torch.empty((micro * self.mb,) + tuple(out_shape), dtype=dtype, device=self.device)
        self.y_all = torch.empty((n_total,) + tuple(out_shape), dtype=dtype, device=self.device)
        self.cuda = self.device.type == "cuda"
        self.comm = torch.cuda.Stream(self.device) if self.cuda else None

    def global_images(self):
        """Global indices of this rank's images, in the order forward() expects them."""
        return [n for a, b in self.ranges for n in range(a, b)]

    def forward(self, x_local, gather=True):
        import torch
        import torch.distributed as dist
        mb, W = self.mb, self.world
        done = []
        for i in range(self.micro):
            xi = x_local[i * mb:(i + 1) * mb]
            yi = self.y_local[i * mb:(i + 1) * mb]
            self.compute(xi, yi)
            if not gather:
                continue
            dst = self.y_all[i * W * mb:(i + 1) * W * mb]
            coll = W > 1 or (dist.is_available() and dist.is_initialized())   # (world 1 under torchrun: NCCL too)
            if self.cuda:
                ev = torch.cuda.Event()
                ev.record()
                self.comm.wait_event(ev)
                with torch.cuda.stream(self.comm):
                    if coll:
                        dist.all_gather_into_tensor(dst, yi, group=self.group)
                    else:
                        dst.copy_(yi)
                yi.record_stream(self.comm)
            else:
                if coll:
                    done.append(dist.all_gather_into_tensor(dst, yi, group=self.group, async_op=True))
                else:
                    dst.copy_(yi)
        for w in done:
            w.wait()
        if gather and self.cuda:
            torch.cuda.current_stream(self.device).wait_stream(self.comm)
        return self.y_all if gather else self.y_local


def env_rank():
    """(rank, local_rank, world) from the torchrun environment (defaults: single process)."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("LOCAL_RANK", "0")),
            int(os.environ.get("WORLD_SIZE", "1")))


# ------------------------------------------------------------------------------------------------------------
# Spatial (D-slab) sharding of one large 3-D volume with a brick-plane halo exchange.
#
# The paper runs one volume per A100 (L758-762) and cites halo exchange between GPUs only as related work
# (DistDL / DistConv, L1690-1694).  Here rank r owns depth planes [r*D/g, (r+1)*D/g) and, before a merged chain
# of stride-1 layers, receives `halo` = sum of the chain's depth paddings planes from each neighbour, rounded up
# to whole brick planes.  It then runs the unchanged merged plan on its extended slab: every output position of
# its own planes depends only on input positions inside the extended slab (the padded-brick region argument of
# Fig 4 applied to the slab faces), and the true volume faces keep their zero padding.
# Brick planes (fixed brick-depth index, N = 1) are contiguous in the bricked layout, so the exchange is two
# contiguous byte ranges per neighbour: no pack / unpack kernels.
# ------------------------------------------------------------------------------------------------------------
def chain_depth_halo(layers) -> int:
    """Depth halo (planes) a merged chain of stride-1 layers needs on each slab face: sum of max(pad, k-1-pad)."""
    h = 0
    for l in layers:
        if l["stride"][0] != 1:
            raise ValueError("spatial sharding needs stride 1 along the sharded (depth) dimension")
        k, p = l["k"][0], l["pad"][0]
        h += max(p, k - 1 - p)
    return h


class SlabGeometry:
    """Own / extended depth range of `rank` and its halo brick planes (all in planes of depth Bd)."""

    def __init__(self, D: int, Bd: int, halo: int, rank: int, world: int):
        if world <= 0 or not (0 <= rank < world):
            raise ValueError("bad rank/world")
        if D % world or (D // world) % Bd:
            raise ValueError(f"depth {D} must split into {world} slabs of whole {Bd}-plane bricks")
        own = D // world
        hp = -(-halo // Bd)                      # halo brick planes per face
        if world > 1 and hp * Bd > own:
            raise ValueError(f"halo {halo} exceeds the slab depth {own}: neighbours only exchange with neighbours")
        self.D, self.Bd, self.rank, self.world = D, Bd, rank, world
        self.own = own
        self.lo, self.hi = rank * own, (rank + 1) * own
        self.halo_planes = hp
        self.lo_planes = hp if rank > 0 else 0          # halo brick planes below (from rank - 1)
        self.hi_planes = hp if rank < world - 1 else 0  # halo brick planes above (from rank + 1)
        self.own_planes = own // Bd
        self.ext_lo = self.lo - self.lo_planes * Bd
        self.ext_D = own + (self.lo_planes + self.hi_planes) * Bd

    def own_slice(self, plane_bytes: int) -> slice:
        """Byte range of the own planes inside the extended bricked buffer."""
        return slice(self.lo_planes * plane_bytes, (self.lo_planes + self.own_planes) * plane_bytes)

    def exchange_ranges(self, plane_bytes: int):
        """[(peer, send byte range, recv byte range)] of the halo exchange, for both neighbours."""
        P, a, o, b, hp = plane_bytes, self.lo_planes, self.own_planes, self.hi_planes, self.halo_planes
        out = []
        if self.rank > 0:   # my first hp own planes are rank-1's upper halo; my lower halo is its last hp planes
            out.append((self.rank - 1, slice(a * P, (a + hp) * P), slice(0, a * P)))
        if self.rank < self.world - 1:
            out.append((self.rank + 1, slice((a + o - hp) * P, (a + o) * P), slice((a + o) * P, (a + o + b) * P)))
        return out


def halo_exchange(ext, plane_bytes: int, geo: SlabGeometry, group=None):
    """Exchange the halo brick planes of a 1-D uint8 extended bricked buffer with both neighbours
    (torch.distributed point-to-point: NCCL over NVLink on GPUs, gloo on CPU)."""
    import torch.distributed as dist
    ops = []
    for peer, snd, rcv in geo.exchange_ranges(plane_bytes):
        ops.append(dist.P2POp(dist.isend, ext[snd], peer, group))
        ops.append(dist.P2POp(dist.irecv, ext[rcv], peer, group))
    if ops:
        for r in dist.batch_isend_irecv(ops):
            r.wait()


def halo_exchange_local(exts, plane_bytes: int, geos):
    """Single-process emulation of halo_exchange for all ranks at once (tests / one-GPU verification)."""
    for geo, ext in zip(geos, exts):
        for peer, _snd, rcv in geo.exchange_ranges(plane_bytes):
            # what `peer` sends to this rank
            for p2, snd2, _r2 in geos[peer].exchange_ranges(plane_bytes):
                if p2 == geo.rank:
                    ext[rcv].copy_(exts[peer][snd2])


class SpatialRunner:
    """One rank's share of a spatially sharded merged chain over one 3-D volume (N = 1).

    forward(x_own) takes this rank's dense [1, C, D/g, H, W] input slab and returns its dense output slab;
    in between: brickify into the extended buffer, halo exchange, the merged plan on the extended slab,
    unbrickify of the own planes.  `exchange` defaults to halo_exchange (torch.distributed).
    """

    def __init__(self, layers, weights, biases, C, D, H, W, brick, dtype, rank, world, device="cuda",
                 group=None, mode=None, **opt_kw):
        from . import engine
        self.geo = SlabGeometry(D, brick[1], chain_depth_halo(layers), rank, world)
        self.group = group
        self.plan = engine.Plan(layers, weights, biases, 1, C, self.geo.ext_D, H, W, 3, dtype, brick,
                                opts=engine.default_opts(**opt_kw) if opt_kw else None, device=device)
        if mode is not None:
            self.plan.set_mode(mode)
        cout = self.plan.out_layout.C
        self.own_in = engine.make_layout(3, 1, C, self.geo.own, H, W, brick, self.plan.dtype)
        self.own_out = engine.make_layout(3, 1, cout, self.geo.own, H, W, brick, self.plan.dtype)
        nbd_ext = self.geo.ext_D // brick[1]
        self.in_plane = int(self.plan.in_layout.total_bytes) // nbd_ext
        self.out_plane = int(self.plan.out_layout.total_bytes) // nbd_ext
        self.xb = self.plan.alloc_bricked(self.plan.in_layout)
        self.yb = self.plan.alloc_bricked(self.plan.out_layout)

    def load(self, x_own, stream=None):
        """Brickify the own input slab into the middle planes of the extended buffer."""
        self.plan.brickify(x_own, out=self.xb[self.geo.own_slice(self.in_plane)], layout=self.own_in, stream=stream)

    def exchange(self):
        halo_exchange(self.xb, self.in_plane, self.geo, self.group)

    def compute(self, out=None, stream=None):
        self.plan.run(self.xb, self.yb, stream=stream)
        return self.plan.unbrickify(self.yb[self.geo.own_slice(self.out_plane)], layout=self.own_out, out=out,
                                    stream=stream)

    def forward(self, x_own, out=None, stream=None):
        self.load(x_own, stream=stream)
        self.exchange()
        return self.compute(out=out, stream=stream)
