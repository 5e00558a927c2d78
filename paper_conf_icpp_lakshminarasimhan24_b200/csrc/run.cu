// Execution entry points of the C ABI: prepare (weight packing, memo-table reset), run a subgraph,
// run the whole graph, memo counters.  Host code; every step of the path runs in our kernels.
#include <cuda_runtime.h>

#include <cstdlib>
#include <string>
#include <vector>

#include "internal.h"
#include "kernels/common.cuh"

namespace bdl {
bdl_status launch_pack_f32(const bdl_layer &l, int dtype, float *w_out, float *b_out, cudaStream_t s);
bdl_status launch_brick_subgraph(bdl_plan *p, const Subgraph &sg, const TView &in, const TView &out,
                                 const std::vector<TView> &res_views, unsigned char *ws, cudaStream_t s,
                                 int *launches);
bdl_status launch_pack_tc(const bdl_layer &l, void *w_out, cudaStream_t s);
bdl_status launch_tc_subgraph(bdl_plan *p, Subgraph &sg, const TView &in, const TView &out,
                              const TView *res, unsigned char *ws, cudaStream_t s, int *launches);
bdl_status launch_ws_subgraph(bdl_plan *p, Subgraph &sg, const TView &in, const TView &out, const TView *res,
                              unsigned char *wsp, cudaStream_t s, int *launches, bool unmerged, void *dense);
bdl_status launch_unbrickify(const bdl_layout *l, const void *src, void *dst, cudaStream_t s);
int tc_launches(const bdl_plan *p, const Subgraph &sg);
bdl_status launch_pack_gen(const bdl_plan *p, const Subgraph &sg, int j, void *w_out, cudaStream_t s);
bdl_status launch_gen_subgraph(bdl_plan *p, Subgraph &sg, const std::vector<TView> &srcv, const TView &out,
                               const std::vector<TView> &res, unsigned char *wsp, cudaStream_t s, int *launches);
int gen_launches(const bdl_plan *p, const Subgraph &sg);

static void *tensor_ptr(const bdl_plan *p, int t, const void *in_b, void *out_b, unsigned char *ws) {
    const Tensor &T = p->tensors[t];
    if (T.ws_off >= 0) return ws + T.ws_off;
    if (T.producer == -1) return const_cast<void *>(in_b);
    return out_b;
}
}  // namespace bdl

using namespace bdl;

extern "C" {

bdl_status bdl_plan_prepare(bdl_plan *p, void *workspace, void *stream) {
    if (!p) return fail(BDL_EINVAL, "bdl_plan_prepare: plan is NULL");
    if (!workspace && p->ws_bytes > 0) return fail(BDL_EINVAL, "bdl_plan_prepare: workspace is NULL");
    if (((uintptr_t)workspace) % 256) return fail(BDL_EINVAL, "bdl_plan_prepare: workspace must be 256-byte aligned");
    unsigned char *ws = (unsigned char *)workspace;
    cudaStream_t s = (cudaStream_t)stream;
    for (auto &L : p->layers) {
        if (L.L.kind != BDL_OP_CONV) continue;
        bdl_status st = launch_pack_f32(L.L, p->in_layout.dtype, (float *)(ws + L.w_off), (float *)(ws + L.b_off), s);
        if (st != BDL_OK) return st;
    }
    for (auto &sg : p->sgs) {
        for (int j = sg.first; j <= sg.last; j++) {
            const Layer &L = p->layers[j];
            if (L.gen_w_off >= 0) {
                bdl_status st = launch_pack_gen(p, sg, j - sg.first, ws + L.gen_w_off, s);
                if (st != BDL_OK) return st;
            }
            if (L.tc_w_off < 0) continue;
            bdl_status st = sg.kernel == KERNEL_TC_GEN ? launch_pack_gen(p, sg, j - sg.first, ws + L.tc_w_off, s)
                                                       : launch_pack_tc(L.L, ws + L.tc_w_off, s);
            if (st != BDL_OK) return st;
        }
    }
    for (auto &sg : p->sgs) {
        if (sg.order_off >= 0)
            cudaMemcpyAsync(ws + sg.order_off, sg.order_host.data(), sg.norder * 4, cudaMemcpyHostToDevice, s);
        cudaMemsetAsync(ws + sg.status_off, 0, sg.ntasks_total * 4, s);
        cudaMemsetAsync(ws + sg.counter_off, 0, 128, s);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(BDL_ECUDA, std::string("bdl_plan_prepare: ") + cudaGetErrorString(e));
    p->prepared = true;
    p->prepared_ws = workspace;
    return BDL_OK;
}

}  // extern "C"

// Run subgraph i; dense != NULL (last subgraph only): write the graph output as dense NC(D)HW there when the
// subgraph's kernel can (*dense_done = 1), else into out_bricked as usual (*dense_done = 0).
static bdl_status run_subgraph_impl(bdl_plan *p, int32_t i, const void *in_bricked, void *out_bricked, void *workspace,
                                    void *stream, void *dense, int *dense_done) {
    if (dense_done) *dense_done = 0;
    if (!p || i < 0 || i >= (int)p->sgs.size()) return fail(BDL_EINVAL, "bdl_run_subgraph: bad plan or index");
    if (!p->prepared || p->prepared_ws != workspace)
        return fail(BDL_EINVAL, "bdl_run_subgraph: call bdl_plan_prepare with this workspace first");
    if (!in_bricked || !out_bricked) return fail(BDL_EINVAL, "bdl_run_subgraph: NULL tensor");
    unsigned char *ws = (unsigned char *)workspace;
    cudaStream_t s = (cudaStream_t)stream;
    Subgraph &sg = p->sgs[i];
    const Tensor &tin = p->tensors[sg.in_tensor];
    const Tensor &tout = p->tensors[sg.out_tensor];
    TView vin = make_view(tin.layout, tensor_ptr(p, sg.in_tensor, in_bricked, out_bricked, ws));
    TView vout = make_view(tout.layout, tensor_ptr(p, sg.out_tensor, in_bricked, out_bricked, ws));
    std::vector<TView> res(sg.last - sg.first + 1);
    const TView *tc_res = nullptr;
    for (size_t j = 0; j < res.size(); j++) {
        int t = sg.res_tensor[j];
        if (t < 0) continue;
        res[j] = make_view(p->tensors[t].layout, tensor_ptr(p, t, in_bricked, out_bricked, ws));
        tc_res = &res[j];
    }
    int launches = 0;
    const int kern = effective_kernel(sg);
    if (kern == KERNEL_TC_GEN) {
        std::vector<TView> srcv(sg.last - sg.first + 1);   // external inputs per layer (graph branches)
        for (size_t j = 0; j < srcv.size(); j++) {
            const int t = sg.src_tensor[j];
            if (t >= 0) srcv[j] = make_view(p->tensors[t].layout, tensor_ptr(p, t, in_bricked, out_bricked, ws));
        }
        return launch_gen_subgraph(p, sg, srcv, vout, res, ws, s, &launches);
    }
    if (kern == KERNEL_TC_BAND) {
        const bool single = sg.first == sg.last;
        if (sg.mode == BDL_MODE_PADDED && !single && sg.gen_padded) {
            std::vector<TView> srcv(sg.last - sg.first + 1);
            srcv[0] = vin;
            return launch_gen_subgraph(p, sg, srcv, vout, res, ws, s, &launches);
        }
        if (sg.mode == BDL_MODE_PADDED && !single) return launch_tc_subgraph(p, sg, vin, vout, tc_res, ws, s, &launches);
        if (dense && dense_done) *dense_done = 1;
        return launch_ws_subgraph(p, sg, vin, vout, tc_res, ws, s, &launches, sg.mode == BDL_MODE_UNMERGED || single,
                                  dense);
    }
    return launch_brick_subgraph(p, sg, vin, vout, res, ws, s, &launches);
}

extern "C" {

bdl_status bdl_run_subgraph(bdl_plan *p, int32_t i, const void *in_bricked, void *out_bricked, void *workspace,
                            void *stream) {
    return run_subgraph_impl(p, i, in_bricked, out_bricked, workspace, stream, nullptr, nullptr);
}

bdl_status bdl_run_dense(bdl_plan *p, const void *in_bricked, void *out_dense, void *workspace, void *stream) {
    if (!p || !out_dense) return fail(BDL_EINVAL, "bdl_run_dense: NULL argument");
    if (!p->prepared || p->prepared_ws != workspace)
        return fail(BDL_EINVAL, "bdl_run_dense: call bdl_plan_prepare with this workspace first");
    unsigned char *ws = (unsigned char *)workspace;
    void *final_b = ws + p->final_off;   // the bricked graph output, when the last kernel cannot write dense
    const int n = (int)p->sgs.size();
    for (int i = 0; i < n; i++) {
        int done = 0;
        bdl_status st = run_subgraph_impl(p, i, in_bricked, final_b, workspace, stream, i == n - 1 ? out_dense : nullptr,
                                          &done);
        if (st != BDL_OK) return st;
        if (i == n - 1 && !done) return bdl_unbrickify(&p->out_layout, final_b, out_dense, stream);
    }
    return BDL_OK;
}

bdl_status bdl_run(bdl_plan *p, const void *in_bricked, void *out_bricked, void *workspace, void *stream) {
    if (!p) return fail(BDL_EINVAL, "bdl_run: plan is NULL");
    for (int i = 0; i < (int)p->sgs.size(); i++) {
        bdl_status st = bdl_run_subgraph(p, i, in_bricked, out_bricked, workspace, stream);
        if (st != BDL_OK) return st;
    }
    return BDL_OK;
}

int32_t bdl_plan_launches_per_run(const bdl_plan *p) {
    if (!p) return 0;
    int n = 0;
    for (auto &sg : p->sgs) {
        int L = sg.last - sg.first + 1;
        const int k = effective_kernel(sg);
        if (k == KERNEL_TC_BAND) n += tc_launches(p, sg);
        else if (k == KERNEL_TC_GEN) n += gen_launches(p, sg);
        else n += (sg.mode == BDL_MODE_UNMERGED || L == 1) ? L : 1;
    }
    return n;
}

bdl_status bdl_plan_counters(const bdl_plan *p, int32_t i, const void *workspace, void *stream, uint64_t out[4]) {
    if (!p || i < 0 || i >= (int)p->sgs.size() || !workspace || !out) return fail(BDL_EINVAL, "bdl_plan_counters: bad args");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e = cudaMemcpyAsync(out, (const unsigned char *)workspace + p->sgs[i].counter_off, 32,
                                    cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return fail(BDL_ECUDA, std::string("bdl_plan_counters: ") + cudaGetErrorString(e));
    return BDL_OK;
}

}  // extern "C"
