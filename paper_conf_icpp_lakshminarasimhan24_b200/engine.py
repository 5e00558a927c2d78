"""High-level Python API over the C ABI: build a plan for a layer graph, own the device workspace,
brickify -> merged execution -> unbrickify.  PyTorch provides device memory and streams only;
all computation happens in libbrickdl.so's kernels.
"""
from __future__ import annotations

import ctypes

import torch

from . import (BDL_BF16, BDL_F32, BDL_MODE_AUTO, BDL_NO_RESIDUAL, BDL_OP_CONV, BDL_OP_MAXPOOL, KERNEL_NAMES,
               MODE_NAMES, bdl_layer, bdl_layout, bdl_plan_opts, check, lib)

_TORCH_DTYPE = {BDL_F32: torch.float32, BDL_BF16: torch.bfloat16}


def make_layout(nsp, N, C, D, H, W, brick, dtype):
    lo = bdl_layout()
    Bn, Bd, Bh, Bw = brick
    check(lib().bdl_layout_init(ctypes.byref(lo), nsp, N, C, D, H, W, Bn, Bd, Bh, Bw, dtype))
    return lo


def default_opts(**kw):
    o = bdl_plan_opts()
    lib().bdl_plan_opts_default(ctypes.byref(o))
    for k, v in kw.items():
        if k == "bcand":
            for i, b in enumerate(v):
                o.bcand[i] = b
        else:
            setattr(o, k, v)
    return o


def _stream_handle(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


class Plan:
    """A partitioned, prepared layer graph (workloads.make_layers format).

    weights: list of float tensors [Co, Ci, kd, kh, kw] (or None for pools); biases: list of [Co].
    With device=None the plan is built host-only (static analysis without a GPU; run() unavailable).
    """

    def __init__(self, layers, weights, biases, N, C, D, H, W, nsp, dtype, brick, opts=None,
                 device="cuda", brickmap=None):
        self.dtype = BDL_BF16 if dtype in ("bf16", BDL_BF16) else BDL_F32
        self.tdtype = _TORCH_DTYPE[self.dtype]
        self.nsp = nsp
        self.device = device
        self.in_layout = make_layout(nsp, N, C, D, H, W, brick, self.dtype)
        self._keep = []
        if brickmap is not None and device is not None:
            bm = torch.as_tensor(brickmap, dtype=torch.int32).to(device).contiguous()
            self._keep.append(bm)
            self.in_layout.brickmap = bm.data_ptr()
        arr = (bdl_layer * len(layers))()
        for i, l in enumerate(layers):
            a = arr[i]
            a.kind = BDL_OP_CONV if l["kind"] == "conv" else BDL_OP_MAXPOOL
            a.cin, a.cout = l["cin"], l["cout"]
            for d in range(3):
                a.k[d], a.stride[d], a.pad[d] = l["k"][d], l["stride"][d], l["pad"][d]
                a.dil[d] = l.get("dil", (1, 1, 1))[d]
            a.groups = l.get("groups", 1)
            a.transposed = 1 if l.get("transposed") else 0
            a.relu = int(l["relu"])
            a.input = l["input"]
            a.residual = BDL_NO_RESIDUAL if l["residual"] is None else l["residual"]
            if a.kind == BDL_OP_CONV:
                if device is None:
                    a.w, a.bias = 1, 1   # host-only planning: pointers are not dereferenced
                else:
                    w = weights[i].permute(0, 2, 3, 4, 1).contiguous().to(device=device, dtype=self.tdtype)
                    b = biases[i].to(device=device, dtype=torch.float32).contiguous()
                    self._keep += [w, b]
                    a.w, a.bias = w.data_ptr(), b.data_ptr()
        self._layers = arr
        self.opts = opts if opts is not None else default_opts()
        h = ctypes.c_void_p()
        check(lib().bdl_graph_partition(arr, len(layers), ctypes.byref(self.in_layout), ctypes.byref(self.opts),
                                        ctypes.byref(h)))
        self.h = h
        self.out_layout = bdl_layout()
        check(lib().bdl_plan_out_layout(h, ctypes.byref(self.out_layout)))
        self.ws = None
        if device is not None:
            nbytes = int(lib().bdl_plan_workspace_bytes(h))
            self.ws = torch.empty(max(nbytes, 256) + 256, dtype=torch.uint8, device=device)
            self.ws_ptr = (self.ws.data_ptr() + 255) // 256 * 256
            self.prepare()

    # ---------------------------------------------------------------- plan introspection
    def __del__(self):
        try:
            if getattr(self, "h", None):
                lib().bdl_plan_destroy(self.h)
                self.h = None
        except Exception:
            pass

    def prepare(self, stream=None):
        # (re)packs weights from the staged device copies kept in self._keep
        check(lib().bdl_plan_prepare(self.h, ctypes.c_void_p(self.ws_ptr), _stream_handle(stream)))

    @property
    def num_subgraphs(self):
        return lib().bdl_plan_num_subgraphs(self.h)

    def subgraphs(self):
        out = []
        for i in range(self.num_subgraphs):
            f, la, m, b, k = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
            d = ctypes.c_double()
            check(lib().bdl_plan_subgraph(self.h, i, ctypes.byref(f), ctypes.byref(la), ctypes.byref(m),
                                          ctypes.byref(b), ctypes.byref(d), ctypes.byref(k)))
            df, rho, mm, tb = ctypes.c_double(), ctypes.c_int64(), ctypes.c_int32(), ctypes.c_int32()
            check(lib().bdl_plan_subgraph_model(self.h, i, ctypes.byref(df), ctypes.byref(rho), ctypes.byref(mm),
                                                ctypes.byref(tb)))
            out.append(dict(first=f.value, last=la.value, mode=MODE_NAMES.get(m.value, m.value),
                            mode_id=m.value, model_brick=b.value, delta=d.value, delta_first=df.value,
                            rho=rho.value, mode_model=MODE_NAMES.get(mm.value, mm.value),
                            kernel=KERNEL_NAMES[k.value], tc_band=tb.value,
                            cta_pair=bool(lib().bdl_plan_subgraph_cta_pair(self.h, i))))
        return out

    def set_mode(self, mode, i=None):
        """mode: 'padded' | 'memoized' | 'unmerged' | 'auto' (all subgraphs, or subgraph i)."""
        ids = {"auto": 0, "padded": 1, "memoized": 2, "unmerged": 3}
        m = ids[mode] if isinstance(mode, str) else mode
        for j in ([i] if i is not None else range(self.num_subgraphs)):
            check(lib().bdl_plan_set_mode(self.h, j, m))
        if self.ws is not None:
            self.prepare()

    @property
    def launches_per_run(self):
        return lib().bdl_plan_launches_per_run(self.h)

    # ---------------------------------------------------------------- execution
    def alloc_bricked(self, layout):
        return torch.empty(int(layout.total_bytes), dtype=torch.uint8, device=self.device)

    def brickify(self, x, out=None, layout=None, stream=None):
        layout = layout if layout is not None else self.in_layout
        x = x.to(device=self.device, dtype=self.tdtype).contiguous()
        out = out if out is not None else self.alloc_bricked(layout)
        check(lib().bdl_brickify(ctypes.byref(layout), ctypes.c_void_p(x.data_ptr()),
                                 ctypes.c_void_p(out.data_ptr()), _stream_handle(stream)))
        return out

    def unbrickify(self, b, layout=None, out=None, stream=None):
        layout = layout if layout is not None else self.out_layout
        shape = (layout.N, layout.C, layout.D, layout.H, layout.W)
        out = out if out is not None else torch.empty(shape, dtype=self.tdtype, device=self.device)
        check(lib().bdl_unbrickify(ctypes.byref(layout), ctypes.c_void_p(b.data_ptr()),
                                   ctypes.c_void_p(out.data_ptr()), _stream_handle(stream)))
        return out

    def run(self, bricked_in, bricked_out=None, stream=None):
        bricked_out = bricked_out if bricked_out is not None else self.alloc_bricked(self.out_layout)
        check(lib().bdl_run(self.h, ctypes.c_void_p(bricked_in.data_ptr()), ctypes.c_void_p(bricked_out.data_ptr()),
                            ctypes.c_void_p(self.ws_ptr), _stream_handle(stream)))
        return bricked_out

    def run_subgraph(self, i, bricked_in, bricked_out, stream=None):
        """Run subgraph i alone (its input/output tensors: graph input/output buffers or workspace)."""
        check(lib().bdl_run_subgraph(self.h, i, ctypes.c_void_p(bricked_in.data_ptr()),
                                     ctypes.c_void_p(bricked_out.data_ptr()), ctypes.c_void_p(self.ws_ptr),
                                     _stream_handle(stream)))

    def run_dense(self, bricked_in, out=None, stream=None):
        """Merged execution writing the dense NC(D)HW output (bdl_run_dense: unbrickify fused into the last
        subgraph's epilogue where its kernel supports it)."""
        lo = self.out_layout
        out = out if out is not None else torch.empty((lo.N, lo.C, lo.D, lo.H, lo.W), dtype=self.tdtype,
                                                      device=self.device)
        check(lib().bdl_run_dense(self.h, ctypes.c_void_p(bricked_in.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                  ctypes.c_void_p(self.ws_ptr), _stream_handle(stream)))
        return out

    def forward(self, x, stream=None):
        """Dense NC(D)HW -> dense output: brickify, every merged subgraph, unbrickify."""
        return self.unbrickify(self.run(self.brickify(x, stream=stream), stream=stream), stream=stream)

    def forward_into(self, x, out, stream=None):
        """forward() into a caller-owned dense output tensor (brick buffers are allocated once and reused)."""
        if getattr(self, "_fw_xb", None) is None:
            self._fw_xb = self.alloc_bricked(self.in_layout)
            self._fw_yb = self.alloc_bricked(self.out_layout)
        self.brickify(x, out=self._fw_xb, stream=stream)
        return self.run_dense(self._fw_xb, out=out, stream=stream)

    def counters(self, i=0, stream=None):
        arr = (ctypes.c_uint64 * 4)()
        check(lib().bdl_plan_counters(self.h, i, ctypes.c_void_p(self.ws_ptr), _stream_handle(stream), arr))
        return dict(computed=arr[0], cas_ok=arr[1], cas_fail=arr[2], spins=arr[3])


def plan_from_workload(wl, device="cuda", **opt_kw):
    """Plan for a workloads.make_workload(...) dict."""
    opts = default_opts(**opt_kw) if opt_kw else None
    return Plan(wl["layers"], wl["weights"], wl["biases"], wl["N"], wl["C"], wl["D"], wl["H"], wl["W"],
                wl["nsp"], wl["dtype"], wl["brick"], opts=opts, device=device)


class HostPipeline:
    """Pipelined host-to-host inference through a Plan (serving path).

    Each request is a dense NC(D)HW tensor in pinned HOST memory.  Request k runs H2D copy -> brickify ->
    merged subgraphs -> unbrickify -> D2H copy; the H2D of request k+1 and the D2H of request k-1 overlap
    the merged execution of request k on three CUDA streams, with `slots` device/host buffer pairs.  All
    computation is the plan's own kernels; PyTorch provides the streams, events and pinned buffers.
    """

    def __init__(self, plan, slots=2):
        self.plan = plan
        self.slots = slots
        dev = plan.device
        lo, li = plan.out_layout, plan.in_layout
        self.in_shape = (li.N, li.C, li.D, li.H, li.W)
        self.out_shape = (lo.N, lo.C, lo.D, lo.H, lo.W)
        self.x_dev = [torch.empty(self.in_shape, dtype=plan.tdtype, device=dev) for _ in range(slots)]
        self.y_dev = [torch.empty(self.out_shape, dtype=plan.tdtype, device=dev) for _ in range(slots)]
        self.y_host = [torch.empty(self.out_shape, dtype=plan.tdtype).pin_memory() for _ in range(slots)]
        self.xb = plan.alloc_bricked(li)
        self.yb = plan.alloc_bricked(lo)
        self.s_h2d, self.s_cmp, self.s_d2h = (torch.cuda.Stream(dev) for _ in range(3))

    def run(self, inputs, on_output=None):
        """Process the pinned host tensors `inputs` in order.  After request k's D2H completes, calls
        on_output(k, y_host) (y_host is valid until the callback returns; its slot is then reused), or, with
        on_output=None, returns the list of output copies.  Returns when everything is done."""
        n, S = len(inputs), self.slots
        # the plan's weight packing / memo-table reset (bdl_plan_prepare) and any caller work were queued on the
        # caller's current stream: every pipeline stream starts after them.  A plan's workspace is used by one
        # stream at a time (its memo tables and run state are shared), so the merged runs stay on s_cmp.
        cur = torch.cuda.current_stream(self.plan.device)
        for st in (self.s_h2d, self.s_cmp, self.s_d2h):
            st.wait_stream(cur)
        h2d_done = [torch.cuda.Event() for _ in range(S)]
        x_free = [torch.cuda.Event() for _ in range(S)]
        cmp_done = [torch.cuda.Event() for _ in range(S)]
        d2h_done = [torch.cuda.Event() for _ in range(S)]
        used = [False] * S
        outs = []

        def drain(k):   # hand request k's output to the caller (waits for its D2H)
            d2h_done[k % S].synchronize()
            if on_output is not None:
                on_output(k, self.y_host[k % S])
            else:
                outs.append(self.y_host[k % S].clone())

        for k in range(n):
            sl = k % S
            if used[sl]:
                drain(k - S)                                   # the host slot is reused by request k
            with torch.cuda.stream(self.s_h2d):
                if used[sl]:
                    self.s_h2d.wait_event(x_free[sl])          # brickify of request k - S has read x_dev[sl]
                self.x_dev[sl].copy_(inputs[k], non_blocking=True)
                h2d_done[sl].record(self.s_h2d)
            self.s_cmp.wait_event(h2d_done[sl])
            if used[sl]:
                self.s_cmp.wait_event(d2h_done[sl])            # D2H of request k - S has read y_dev[sl]
            self.plan.brickify(self.x_dev[sl], out=self.xb, stream=self.s_cmp)
            x_free[sl].record(self.s_cmp)
            self.plan.run_dense(self.xb, out=self.y_dev[sl], stream=self.s_cmp)
            cmp_done[sl].record(self.s_cmp)
            with torch.cuda.stream(self.s_d2h):
                self.s_d2h.wait_event(cmp_done[sl])
                self.y_host[sl].copy_(self.y_dev[sl], non_blocking=True)
                d2h_done[sl].record(self.s_d2h)
            used[sl] = True
        for k in range(max(0, n - S), n):
            drain(k)
        return None if on_output is not None else outs
