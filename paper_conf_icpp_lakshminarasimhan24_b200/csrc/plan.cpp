// Static analysis (§3.3): graph partitioning (L603-626), padded-vs-memoized mode choice
// by padding data growth Delta (L628-647), brick-size model rho/tau (L649-662), and the
// workspace layout of a plan.  Host-only C++.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <new>
#include <string>

#include "internal.h"

namespace bdl {

// Output extent of a layer along one dim: floor((I + 2p - (k-1) - 1)/s) + 1; transposed conv (I-1)s - 2p + d(k-1) + 1.
static int out_extent(int I, int k, int s, int p, int d, int tr = 0) {
    return tr ? (I - 1) * s - 2 * p + d * (k - 1) + 1 : (I + 2 * p - d * (k - 1) - 1) / s + 1;
}
static int64_t fdiv(int64_t a, int64_t b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }   // floor(a / b), b > 0
static int64_t cdiv(int64_t a, int64_t b) { return -fdiv(-a, b); }                            // ceil(a / b)
// Input extent of one window, d(k-1) + 1.  Layers are normalized at partition time (dil >= 1).
static int keff(const bdl_layer &l, int dim) { return (l.dil[dim] > 1 ? l.dil[dim] : 1) * (l.k[dim] - 1) + 1; }

static int64_t align_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

// ---------------------------------------------------------------------------------------------
// Region analysis (Fig 4): reverse traversal from an output brick region [a, b) of the
// subgraph's last layer; returns per layer the INPUT region of that layer (unclipped) along one dim.
// in_lo[j], in_hi[j] for j = 0..L-1 (layer first+j).  The traversal follows the graph, not the listing:
// a layer's input region is added to the output region needed of the layer it reads, and its output
// region to that of its residual's producer (branches merge by interval hull), so a projection
// shortcut or a skip connection inside the subgraph is sized by its real consumers.  For a chain this
// is the paper's Fig 4 recursion I = s(O-1) + k.  halo = false: the halo-free region s(O-1) + min(k, s) (windows
// that do not overlap: a pool of k = s needs B x s without padding, L456-458), so Delta >= 0.
static void regions_dag(const std::vector<Layer> &ly, int first, int last, int dim, int64_t a, int64_t b, bool halo,
                        std::vector<int64_t> &in_lo, std::vector<int64_t> &in_hi) {
    int L = last - first + 1;
    std::vector<int64_t> olo(L, INT64_MAX), ohi(L, INT64_MIN);
    olo[L - 1] = a;
    ohi[L - 1] = b;
    in_lo.assign(L, 0);
    in_hi.assign(L, 0);
    for (int j = L - 1; j >= 0; j--) {
        if (olo[j] >= ohi[j]) continue;   // output not needed inside the subgraph (a live-out only)
        const bdl_layer &l = ly[first + j].L;
        int k = dim == 0 ? 1 : keff(l, dim - 1), s = dim == 0 ? 1 : l.stride[dim - 1], p = dim == 0 ? 0 : l.pad[dim - 1];
        int64_t lo, hi;
        if (dim > 0 && l.kind == BDL_OP_CONV && l.transposed) {
            // transposed conv: input i reaches outputs s*i - p + d*t, t < k: the inputs reaching [olo, ohi)
            const int kk = halo ? k : std::min(k, s), pp = halo ? p : 0;
            lo = cdiv(olo[j] + pp - (kk - 1), s);
            hi = fdiv(ohi[j] - 1 + pp, s) + 1;
        } else if (halo) {
            lo = olo[j] * s - p;               // input extent I = s(O-1) + k (Q19)
            hi = (ohi[j] - 1) * s - p + k;
        } else {                               // halo-free: non-overlapping windows of the same stride
            lo = olo[j] * s;
            hi = (ohi[j] - 1) * s + std::min(k, s);
        }
        in_lo[j] = lo;
        in_hi[j] = hi;
        const int src = l.input - first;
        if (src >= 0) {
            olo[src] = std::min(olo[src], lo);
            ohi[src] = std::max(ohi[src], hi);
        }
        if (l.residual != BDL_NO_RESIDUAL && l.residual >= first) {
            const int r = l.residual - first;
            olo[r] = std::min(olo[r], olo[j]);
            ohi[r] = std::max(ohi[r], ohi[j]);
        }
    }
}
static void regions_1d(const std::vector<Layer> &ly, int first, int last, int dim, int64_t a, int64_t b,
                       std::vector<int64_t> &in_lo, std::vector<int64_t> &in_hi) {
    regions_dag(ly, first, last, dim, a, b, true, in_lo, in_hi);
}

// Delta: sum over layers and bricks of the padded input region (clipped at the feature
// map) over the halo-free region, minus 1.  `first_only` gives the alternative reading (first
// layer's input only).  Brick extents B[4] over (n, d, h, w) of the last layer's output.
double compute_delta(const std::vector<Layer> &ly, int first, int last, const int B[4], bool first_only) {
    int L = last - first + 1;
    const Layer &lastL = ly[last];
    std::vector<double> pad_sum(L, 1.0), exact_sum(L, 1.0);
    for (int dim = 0; dim < 4; dim++) {
        int64_t ext_out = lastL.out_ext[dim];
        int64_t nb = (ext_out + B[dim] - 1) / B[dim];
        std::vector<double> ps(L, 0.0), es(L, 0.0);
        for (int64_t i = 0; i < nb; i++) {
            int64_t a = i * B[dim], b = std::min<int64_t>(a + B[dim], ext_out);
            std::vector<int64_t> lo, hi, elo, ehi;
            regions_dag(ly, first, last, dim, a, b, true, lo, hi);
            regions_dag(ly, first, last, dim, a, b, false, elo, ehi);
            for (int j = 0; j < L; j++) {
                int64_t I = ly[first + j].in_ext[dim];
                ps[j] += (double)std::max<int64_t>(0, std::min(hi[j], I) - std::max<int64_t>(lo[j], 0));
                es[j] += (double)std::max<int64_t>(0, std::min(ehi[j], I) - std::max<int64_t>(elo[j], 0));
            }
        }
        for (int j = 0; j < L; j++) {
            pad_sum[j] *= ps[j];
            exact_sum[j] *= es[j];
        }
    }
    double P = 0, E = 0;
    for (int j = 0; j < (first_only ? 1 : L); j++) {
        double c = ly[first + j].L.cin;
        P += c * pad_sum[j];
        E += c * exact_sum[j];
    }
    return E > 0 ? P / E - 1.0 : 0.0;
}

// rho/tau brick-size model (L649-658): rho(B) = prod(blocked dims) / B^n over the candidate set,
// pick the largest rho <= tau (the batch counts as a blocked dim, so rho = #bricks).
int model_brick(const bdl_plan_opts &o, int nsp, const int ext[4], int64_t *rho_out) {
    int best = -1;
    double best_rho = -1;
    int largest = 0;
    for (int i = 0; i < 4; i++) {
        int Bc = o.bcand[i];
        if (Bc <= 0) continue;
        largest = std::max(largest, Bc);
        double rho = (double)ext[0];
        for (int d = 4 - nsp; d < 4; d++) rho *= (double)ext[d] / Bc;
        if (rho <= (double)o.tau && rho > best_rho) {
            best_rho = rho;
            best = Bc;
        }
    }
    if (best < 0) {  // every candidate exceeds tau: the coarsest brick
        best = largest;
        best_rho = (double)ext[0];
        for (int d = 4 - nsp; d < 4; d++) best_rho *= (double)ext[d] / best;
    }
    if (rho_out) *rho_out = (int64_t)std::llround(best_rho);
    return best;
}

static bool is_pool(const Layer &l) { return l.L.kind == BDL_OP_MAXPOOL; }

}  // namespace bdl

namespace bdl {
int tc_band_rows(const bdl_plan *p, const Subgraph &sg, int *smem_out);
int ws_band_rows(const bdl_plan *p, const Subgraph &sg);
std::vector<int> ws_task_order(const bdl_plan *p, const Subgraph &sg);
int gen_conv_layers(const bdl_plan *p, const Subgraph &sg);
int64_t gen_layer_tasks(const bdl_plan *p, const Subgraph &sg, int j);
size_t gen_packed_bytes(const bdl_plan *p, const Subgraph &sg, int j);
std::vector<int> gen_task_order(const bdl_plan *p, const Subgraph &sg);

int64_t gen_scratch_bytes(const bdl_plan *p, const Subgraph &sg);
bool gen_layer_supported(const bdl_plan *p, int layer);

int effective_kernel(const Subgraph &sg) { return sg.kernel; }
}
using namespace bdl;

// ---------------------------------------------------------------------------------------------
// tcgen05 band-kernel eligibility (3x3 stride-1 pad-1 2-D convs, Cin = Cout = C,
// C in {16, 32, 64, 128}, batch brick 1, residual only from the subgraph input at the last layer).

static bool tc_eligible(const bdl_plan *p, const Subgraph &sg) {
    if (p->in_layout.dtype != BDL_BF16) return false;
    if (p->in_layout.Bn != 1 || !sg.chain) return false;
    if (p->in_layout.brickmap) return false;   // the band kernels' TMA rows need the identity BrickMap
    const Layer &f = p->layers[sg.first];
    int C = f.L.cin;
    if (!(C == 16 || C == 32 || C == 64 || C == 128)) return false;
    int nsp = p->in_layout.nsp;
    for (int j = sg.first; j <= sg.last; j++) {
        const bdl_layer &l = p->layers[j].L;
        if (l.kind != BDL_OP_CONV || l.cin != C || l.cout != C || l.groups != 1 || l.transposed) return false;
        if (l.dil[0] != 1 || l.dil[1] != 1 || l.dil[2] != 1) return false;
        for (int d = 0; d < 3; d++) {
            bool spatial = (nsp == 3) || d > 0;
            int k = spatial ? 3 : 1, pp = spatial ? 1 : 0;
            if (l.k[d] != k || l.stride[d] != 1 || l.pad[d] != pp) return false;
        }
        int jj = j - sg.first;
        int rt = sg.res_tensor[jj];
        if (rt >= 0 && !(j == sg.last && rt == sg.in_tensor)) return false;
        if (l.residual != BDL_NO_RESIDUAL && rt < 0) return false;
    }
    int smem = 0;
    // memoized / unmerged run on the warp-specialized kernel (C <= 64); wider chains go to the generic kernel
    return tc_band_rows(p, sg, &smem) > 0 && ws_band_rows(p, sg) > 0;
}

extern "C" {

bdl_status bdl_graph_partition(const bdl_layer *layers, int32_t nlayers, const bdl_layout *in,
                               const bdl_plan_opts *opts_in, bdl_plan **out) {
    if (!layers || nlayers <= 0 || !out) return fail(BDL_EINVAL, "bdl_graph_partition: bad arguments");
    if (!layout_valid(in)) return fail(BDL_EINVAL, "bdl_graph_partition: bad input layout");
    *out = nullptr;
    bdl_plan *p = new (std::nothrow) bdl_plan();
    if (!p) return fail(BDL_ENOMEM, "bdl_graph_partition: out of host memory");
    if (opts_in) p->opts = *opts_in; else bdl_plan_opts_default(&p->opts);
    p->in_layout = *in;

    // device facts (the planner also runs on hosts without a GPU: B200 defaults)
    p->num_sms = 148;
    p->l2_bytes = 126LL << 20;
    int dev_count = 0;
    if (cudaGetDeviceCount(&dev_count) == cudaSuccess && dev_count > 0) {
        int dev = 0, v = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && v > 0) p->num_sms = v;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrL2CacheSize, dev) == cudaSuccess && v > 0) p->l2_bytes = v;
    } else {
        cudaGetLastError();
    }
    if (p->opts.num_sms > 0) p->num_sms = p->opts.num_sms;
    int64_t budget = p->opts.onchip_budget > 0 ? p->opts.onchip_budget : p->l2_bytes;

    // ---- layer shapes
    const int nsp = in->nsp;
    p->layers.resize(nlayers);
    for (int i = 0; i < nlayers; i++) {
        Layer &L = p->layers[i];
        L.L = layers[i];
        for (int d = 0; d < 3; d++) L.L.dil[d] = std::max(1, L.L.dil[d]);
        L.L.groups = std::max(1, L.L.groups);
        const bdl_layer &l = L.L;
        if (l.groups > 1 && (l.kind != BDL_OP_CONV || l.cin % l.groups || l.cout % l.groups)) {
            bdl_plan_destroy(p);
            return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": groups must divide cin and cout (convs only)");
        }
        if (l.transposed && (l.kind != BDL_OP_CONV || l.groups != 1)) {
            bdl_plan_destroy(p);
            return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": transposed convs only (groups = 1)");
        }
        if (l.kind == BDL_OP_MAXPOOL && (l.dil[0] != 1 || l.dil[1] != 1 || l.dil[2] != 1)) {
            bdl_plan_destroy(p);
            return fail(BDL_EUNSUPPORTED, "layer " + std::to_string(i) + ": dilated pooling");
        }
        if (l.kind != BDL_OP_CONV && l.kind != BDL_OP_MAXPOOL) {
            bdl_plan_destroy(p);
            return fail(BDL_EUNSUPPORTED, "layer " + std::to_string(i) + ": unknown op kind");
        }
        if (l.input < -1 || l.input >= i) {
            bdl_plan_destroy(p);
            return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": input must be an earlier layer or -1");
        }
        int cin_expected = l.input == -1 ? (int)in->C : p->layers[l.input].L.cout;
        if (l.cin != cin_expected || l.cout <= 0 || (l.kind == BDL_OP_MAXPOOL && l.cout != l.cin)) {
            bdl_plan_destroy(p);
            return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": channel count mismatch");
        }
        if (l.kind == BDL_OP_CONV && !l.w) {
            bdl_plan_destroy(p);
            return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": conv without weights");
        }
        const int *src = nullptr;
        int gin[4] = {(int)in->N, (int)in->D, (int)in->H, (int)in->W};
        src = l.input == -1 ? gin : p->layers[l.input].out_ext;
        for (int d = 0; d < 4; d++) L.in_ext[d] = src[d];
        L.out_ext[0] = L.in_ext[0];
        for (int d = 0; d < 3; d++) {
            if (l.k[d] <= 0 || l.stride[d] <= 0 || l.pad[d] < 0 || (nsp == 2 && d == 0 && (l.k[0] != 1 || l.stride[0] != 1 || l.pad[0] != 0))) {
                bdl_plan_destroy(p);
                return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": bad kernel/stride/pad");
            }
            L.out_ext[d + 1] = out_extent(L.in_ext[d + 1], l.k[d], l.stride[d], l.pad[d], l.dil[d], l.transposed);
            if (L.out_ext[d + 1] <= 0) {
                bdl_plan_destroy(p);
                return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": empty output");
            }
        }
        if (l.residual != BDL_NO_RESIDUAL) {
            if (l.residual < -1 || l.residual >= i) {
                bdl_plan_destroy(p);
                return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": bad residual index");
            }
            const int *rs = l.residual == -1 ? gin : p->layers[l.residual].out_ext;
            int rc = l.residual == -1 ? (int)in->C : layers[l.residual].cout;
            bool same = rc == l.cout;
            for (int d = 0; d < 4; d++) same = same && rs[d] == L.out_ext[d];
            if (!same) {
                bdl_plan_destroy(p);
                return fail(BDL_EINVAL, "layer " + std::to_string(i) + ": residual shape mismatch");
            }
        }
    }
    const int Bx[4] = {in->Bn, in->Bd, in->Bh, in->Bw};
    // Q8: a brick must be at least the kernel's extent (L741) for the layers of a merged subgraph.
    auto fits_brick = [&](int j) {
        const bdl_layer &l = p->layers[j].L;
        for (int d = 0; d < 3; d++)
            if (keff(l, d) > Bx[d + 1] || l.pad[d] > Bx[d + 1]) return false;
        return true;
    };
    auto consumed_after = [&](int m, int end) {
        for (int j = end + 1; j < nlayers; j++)
            if (p->layers[j].L.input == m || p->layers[j].L.residual == m) return true;
        return false;
    };
    // DAG subgraphs (a layer reading a non-previous layer, a residual produced inside the subgraph, or an inner
    // layer read by a later subgraph) run on the generic tcgen05 kernel, which tracks per-layer producers; the
    // paper ends subgraphs only at pools and normalisations (L620-626), not at branches.
    const bool dag_ok = in->dtype == BDL_BF16 && in->Bn == 1;
    auto range_ok = [&](int first, int end) {
        if (p->opts.max_subgraph_layers > 0 && end - first + 1 > p->opts.max_subgraph_layers) return false;
        if (end - first + 1 > kMaxLayers) return false;
        bool branch = false, all_gen = true;
        for (int j = first; j <= end; j++) {
            if (!fits_brick(j)) return false;
            if (j < end && is_pool(p->layers[j])) return false;                 // pool ends a subgraph (L620-626)
            const int r = p->layers[j].L.residual;
            branch = branch || (j > first && p->layers[j].L.input != j - 1) || (r != BDL_NO_RESIDUAL && r >= first) ||
                     (j < end && consumed_after(j, end));
            if (!(j == end && is_pool(p->layers[j]))) all_gen = all_gen && gen_layer_supported(p, j);
            // bf16: grouped (depthwise) convs run on the CUDA-core kernels, dense ones on the tensor cores: the two
            // do not share a subgraph (the whole subgraph runs on one kernel)
            // (transposed convs too: CUDA-core only)
            auto cc = [&](int q) { return p->layers[q].L.groups > 1 || p->layers[q].L.transposed; };
            if (in->dtype == BDL_BF16 && j > first && p->layers[j].L.kind == BDL_OP_CONV &&
                p->layers[j - 1].L.kind == BDL_OP_CONV && cc(j) != cc(j - 1))
                return false;
        }
        if (branch && !(dag_ok && all_gen)) return false;
        // footprint (L605-614): concurrently resident bricks x padded regions + weights.  The persistent kernels hold
        // one tile's region per SM at a time, so the resident bricks are one per SM.
        int nconc = p->num_sms;
        int64_t fp = 0;
        std::vector<int64_t> lo, hi;
        int64_t vol_sum = 0;
        {
            std::vector<int64_t> ext(end - first + 1, 1);
            for (int d = 0; d < 4; d++) {
                regions_1d(p->layers, first, end, d, 0, Bx[d], lo, hi);
                for (int j = 0; j <= end - first; j++) ext[j] *= (hi[j] - lo[j]);
            }
            for (int j = 0; j <= end - first; j++) vol_sum += ext[j] * p->layers[first + j].L.cin;
        }
        fp = (int64_t)nconc * vol_sum * in->elem_bytes;
        for (int j = first; j <= end; j++) {
            const bdl_layer &l = p->layers[j].L;
            fp += (int64_t)l.cout * (l.cin / l.groups) * l.k[0] * l.k[1] * l.k[2] * in->elem_bytes;
        }
        return fp <= budget;
    };

    // ---- reverse traversal partition (L605-614)
    std::vector<std::pair<int, int>> ranges;
    int end = nlayers - 1;
    while (end >= 0) {
        int first = end;
        while (first - 1 >= 0 && !is_pool(p->layers[first - 1]) && range_ok(first - 1, end)) first--;
        ranges.push_back({first, end});
        end = first - 1;
    }
    std::reverse(ranges.begin(), ranges.end());

    // ---- tensors: graph input, every subgraph output
    Tensor tin;
    tin.producer = -1;
    tin.layout = *in;
    tin.ws_off = -1;
    p->tensors.push_back(tin);
    auto tensor_of = [&](int producer) {
        for (size_t t = 0; t < p->tensors.size(); t++)
            if (p->tensors[t].producer == producer) return (int)t;
        return -1;
    };
    for (auto &r : ranges) {
        Subgraph sg;
        sg.first = r.first;
        sg.last = r.second;
        const Layer &fl = p->layers[sg.first];
        sg.in_tensor = tensor_of(fl.L.input);
        if (sg.in_tensor < 0) {
            bdl_plan_destroy(p);
            return fail(BDL_EINVAL, "partition: subgraph input is not materialized (internal error)");
        }
        bool liveout = false;
        for (int j = sg.first; j <= sg.last; j++) {
            const bdl_layer &l = p->layers[j].L;
            const int src = l.input >= sg.first ? l.input - sg.first : -1;
            sg.src_local.push_back(src);
            int st = -1;
            if (src < 0) {
                st = tensor_of(l.input);
                if (st < 0) {
                    bdl_plan_destroy(p);
                    return fail(BDL_EINVAL, "partition: layer " + std::to_string(j) + " input is not materialized");
                }
            }
            sg.src_tensor.push_back(st);
            if (j > sg.first && src != j - 1 - sg.first) sg.chain = false;
            const int r2 = l.residual;
            if (r2 != BDL_NO_RESIDUAL && r2 >= sg.first) {
                sg.res_local.push_back(r2 - sg.first);
                sg.res_tensor.push_back(-1);
                sg.chain = false;
            } else if (r2 != BDL_NO_RESIDUAL) {
                int t2 = tensor_of(r2);
                if (t2 < 0) {
                    bdl_plan_destroy(p);
                    return fail(BDL_EUNSUPPORTED, "layer " + std::to_string(j) + ": residual source is not materialized");
                }
                sg.res_local.push_back(-1);
                sg.res_tensor.push_back(t2);
            } else {
                sg.res_local.push_back(-1);
                sg.res_tensor.push_back(-1);
            }
        }
        const Layer &ll = p->layers[sg.last];
        Tensor t;
        t.producer = sg.last;
        bdl_layout_init(&t.layout, nsp, ll.out_ext[0], ll.L.cout, ll.out_ext[1], ll.out_ext[2], ll.out_ext[3],
                        in->Bn, in->Bd, in->Bh, in->Bw, in->dtype);
        t.ws_off = 0;
        if (t.layout.N == in->N && t.layout.D == in->D && t.layout.H == in->H && t.layout.W == in->W)
            t.layout.brickmap = in->brickmap;  // same grid: keep the caller's BrickMap
        p->tensors.push_back(t);
        sg.out_tensor = (int)p->tensors.size() - 1;
        // inner layers read by later subgraphs: their memo buffers are materialized tensors
        for (int j = sg.first; j < sg.last; j++) {
            if (!consumed_after(j, sg.last)) continue;
            const Layer &ly = p->layers[j];
            Tensor lt;
            lt.producer = j;
            bdl_layout_init(&lt.layout, nsp, ly.out_ext[0], ly.L.cout, ly.out_ext[1], ly.out_ext[2], ly.out_ext[3],
                            in->Bn, in->Bd, in->Bh, in->Bw, in->dtype);
            lt.ws_off = 0;
            p->tensors.push_back(lt);
            liveout = true;
        }
        if (liveout) sg.chain = false;
        // ---- models
        int ext_in[4];
        for (int d = 0; d < 4; d++) ext_in[d] = fl.in_ext[d];
        sg.model_brick = model_brick(p->opts, nsp, ext_in, &sg.rho);
        if (p->opts.force_brick > 0) sg.model_brick = p->opts.force_brick;   // padded block edge override
        sg.delta = compute_delta(p->layers, sg.first, sg.last, Bx, false);
        sg.delta_first = compute_delta(p->layers, sg.first, sg.last, Bx, true);
        // executed brick = the layout's; the tiny-layer rule (L659-662) uses it
        double rho_exec = (double)ext_in[0];
        int64_t bn = 1;
        for (int d = 4 - nsp; d < 4; d++) {
            rho_exec *= (double)ext_in[d] / Bx[d];
            bn *= Bx[d];
        }
        if (sg.last == sg.first) sg.mode_model = BDL_MODE_UNMERGED;
        else if (rho_exec < (double)bn) sg.mode_model = BDL_MODE_UNMERGED;
        else sg.mode_model = sg.delta > p->opts.delta_threshold ? BDL_MODE_MEMOIZED : BDL_MODE_PADDED;
        // padded mode recomputes a chain per CTA block and materializes only the last layer: a DAG subgraph
        // (branches, inner live-outs) executes memoized instead
        if (!sg.chain && sg.mode_model == BDL_MODE_PADDED) sg.mode_model = BDL_MODE_MEMOIZED;
        sg.mode = p->opts.force_mode != BDL_MODE_AUTO ? p->opts.force_mode : sg.mode_model;
        if (!sg.chain && sg.mode == BDL_MODE_PADDED) sg.mode = BDL_MODE_MEMOIZED;
        p->sgs.push_back(sg);
    }
    p->tensors[p->sgs.back().out_tensor].ws_off = -1;  // graph output is the user's buffer
    p->out_layout = p->tensors[p->sgs.back().out_tensor].layout;
    for (auto &sg : p->sgs) {
        sg.kernel = tc_eligible(p, sg) ? KERNEL_TC_BAND : KERNEL_BRICK;
        if (sg.kernel == KERNEL_BRICK && (sg.gen_layers = gen_conv_layers(p, sg)) > 0) sg.kernel = KERNEL_TC_GEN;
        // band-kernel chains run PADDED mode on the generic kernel (warp-specialized, measured faster on B200 than
        // the synchronous band padded kernel: cfg2 0.195 -> see DESIGN.md §8); same per-element K order, so the
        // modes stay bit-equal
        if (sg.kernel == KERNEL_TC_BAND && sg.last > sg.first && (sg.gen_layers = gen_conv_layers(p, sg)) > 0)
            sg.gen_padded = true;
        if (!sg.chain && sg.kernel != KERNEL_TC_GEN) {
            bdl_plan_destroy(p);
            return fail(BDL_EUNSUPPORTED, "partition: a branched subgraph cannot run on the generic kernel");
        }
    }

    // ---- workspace layout
    int64_t off = 0;
    auto take = [&](int64_t bytes) {
        int64_t o = align_up(off, 256);
        off = o + align_up(bytes, 256);
        return o;
    };
    for (auto &L : p->layers) {
        if (L.L.kind != BDL_OP_CONV) continue;
        int64_t taps = (int64_t)L.L.k[0] * L.L.k[1] * L.L.k[2];
        L.w_off = take(taps * (L.L.cin / L.L.groups) * L.L.cout * 4);
        L.b_off = take((int64_t)L.L.cout * 4);
    }
    for (auto &sg : p->sgs)
        if (sg.kernel == KERNEL_TC_BAND)
            for (int j = sg.first; j <= sg.last; j++) {
                Layer &L = p->layers[j];
                int64_t taps = (int64_t)L.L.k[0] * L.L.k[1] * L.L.k[2];
                L.tc_w_off = take(taps * L.L.cin * L.L.cout * 2);
            }
        else if (sg.kernel == KERNEL_TC_GEN)
            for (int j = 0; j < sg.gen_layers; j++) p->layers[sg.first + j].tc_w_off = take(gen_packed_bytes(p, sg, j));
    for (auto &sg : p->sgs)
        if (sg.gen_padded)
            for (int j = 0; j < sg.gen_layers; j++) p->layers[sg.first + j].gen_w_off = take(gen_packed_bytes(p, sg, j));
    for (size_t t = 1; t < p->tensors.size(); t++)
        if (p->tensors[t].ws_off == 0) p->tensors[t].ws_off = take(p->tensors[t].layout.total_bytes);
    for (auto &sg : p->sgs) {
        int L = sg.last - sg.first + 1;
        sg.memo_off.assign(L, -1);
        sg.task_base.assign(L, 0);
        int64_t words = 0;
        for (int j = 0; j < L; j++) {
            const Layer &ly = p->layers[sg.first + j];
            bdl_layout lo;
            bdl_layout_init(&lo, nsp, ly.out_ext[0], ly.L.cout, ly.out_ext[1], ly.out_ext[2], ly.out_ext[3],
                            in->Bn, in->Bd, in->Bh, in->Bw, in->dtype);
            if (j < L - 1) {
                const int lt = tensor_of(sg.first + j);   // a live-out's buffer is its tensor
                sg.memo_off[j] = lt >= 0 ? p->tensors[lt].ws_off : take(lo.total_bytes);
            }
            sg.task_base[j] = words;
            // memo tags: one per brick, or per band task of the tcgen05 kernels (bands of >= 1 row)
            int64_t w = std::max<int64_t>(lo.nbricks, lo.N * lo.D * lo.H * lo.nb[3]);
            if (sg.kernel == KERNEL_TC_GEN) w = std::max<int64_t>(w, gen_layer_tasks(p, sg, j));
            words += w;
        }
        sg.ntasks_total = words;
        sg.status_off = take(words * 4);
        sg.counter_off = take(16 * 8);   // [0..7] subgraph kernel, [8..15] trailing-pool kernel
        // padded-mode scratch for the CUDA-core kernel: two ping-pong region buffers per CTA
        int64_t maxvol = 1;
        {
            std::vector<int64_t> ext(L, 1);
            std::vector<int64_t> lo, hi;
            for (int d = 0; d < 4; d++) {
                regions_1d(p->layers, sg.first, sg.last, d, 0, Bx[d], lo, hi);
                for (int j = 0; j < L; j++) ext[j] *= (hi[j] - lo[j]);
            }
            // output region of layer j (j < L-1) == input region of layer j+1
            for (int j = 1; j < L; j++) maxvol = std::max(maxvol, ext[j] * (int64_t)p->layers[sg.first + j].L.cin);
        }
        sg.grid = 4 * p->num_sms;
        sg.scratch_slot_floats = align_up(maxvol, 64);
        sg.scratch_off = L > 1 ? take((int64_t)sg.grid * 2 * sg.scratch_slot_floats * 4) : -1;
        if (sg.kernel == KERNEL_TC_BAND) {
            sg.tc_band = tc_band_rows(p, sg, &sg.tc_smem);
            if (int wb = ws_band_rows(p, sg)) sg.tc_band = wb;  // memoized/unmerged band height
            sg.order_host = ws_task_order(p, sg);
            sg.norder = (int64_t)sg.order_host.size();
            sg.order_off = sg.norder ? take(sg.norder * 4) : -1;
        }
        if (sg.gen_padded) {
            if (int64_t sb = gen_scratch_bytes(p, sg)) sg.gen_scr_off = take(sb);
        } else if (sg.kernel == KERNEL_TC_GEN) {
            if (int64_t sb = gen_scratch_bytes(p, sg)) sg.gen_scr_off = take(sb);
            sg.order_host = gen_task_order(p, sg);
            sg.norder = (int64_t)sg.order_host.size();
            sg.order_off = sg.norder ? take(sg.norder * 4) : -1;
        }
    }
    p->final_off = take(p->out_layout.total_bytes);   // bdl_run_dense: bricked output when the last kernel cannot write dense
    p->ws_bytes = align_up(off, 256);
    *out = p;
    return BDL_OK;
}

int32_t bdl_plan_num_subgraphs(const bdl_plan *p) { return p ? (int32_t)p->sgs.size() : 0; }

bdl_status bdl_plan_subgraph(const bdl_plan *p, int32_t i, int32_t *first, int32_t *last, int32_t *mode,
                             int32_t *mbrick, double *delta, int32_t *kernel) {
    if (!p || i < 0 || i >= (int)p->sgs.size()) return fail(BDL_EINVAL, "bdl_plan_subgraph: bad index");
    const Subgraph &s = p->sgs[i];
    if (first) *first = s.first;
    if (last) *last = s.last;
    if (mode) *mode = s.mode;
    if (mbrick) *mbrick = s.model_brick;
    if (delta) *delta = s.delta;
    if (kernel) *kernel = effective_kernel(s);
    return BDL_OK;
}

bdl_status bdl_plan_set_mode(bdl_plan *p, int32_t i, int32_t mode) {
    if (!p || i < 0 || i >= (int)p->sgs.size()) return fail(BDL_EINVAL, "bdl_plan_set_mode: bad index");
    if (mode == BDL_MODE_AUTO) mode = p->sgs[i].mode_model;
    if (mode < BDL_MODE_PADDED || mode > BDL_MODE_UNMERGED) return fail(BDL_EINVAL, "bdl_plan_set_mode: bad mode");
    if (mode == BDL_MODE_PADDED && !p->sgs[i].chain) mode = BDL_MODE_MEMOIZED;   // DAG subgraph: see partition
    p->sgs[i].mode = mode;
    p->prepared = false;
    return BDL_OK;
}

bdl_status bdl_plan_out_layout(const bdl_plan *p, bdl_layout *out) {
    if (!p || !out) return fail(BDL_EINVAL, "bdl_plan_out_layout: NULL");
    *out = p->out_layout;
    return BDL_OK;
}

int64_t bdl_plan_workspace_bytes(const bdl_plan *p) { return p ? p->ws_bytes : 0; }

void bdl_plan_destroy(bdl_plan *p) { delete p; }

// Extra host-side introspection used by tests (not in the header's required set, but C ABI):
// Delta alternative reading and rho of subgraph i.
bdl_status bdl_plan_subgraph_model(const bdl_plan *p, int32_t i, double *delta_first, int64_t *rho,
                                   int32_t *mode_model, int32_t *tc_band) {
    if (!p || i < 0 || i >= (int)p->sgs.size()) return fail(BDL_EINVAL, "bad index");
    const Subgraph &s = p->sgs[i];
    if (delta_first) *delta_first = s.delta_first;
    if (rho) *rho = s.rho;
    if (mode_model) *mode_model = s.mode_model;
    if (tc_band) *tc_band = s.tc_band;
    return BDL_OK;
}

// Region table (Fig 4): input-region extent of each layer of layers [first, last] for an output
// brick of edge `b` along one spatial dim (d = 1..3), interior brick (unclipped).
bdl_status bdl_region_extents(const bdl_layer *layers, int32_t first, int32_t last, int32_t dim, int32_t b,
                              int64_t *ext_out) {
    if (!layers || first < 0 || last < first || dim < 1 || dim > 3 || !ext_out) return fail(BDL_EINVAL, "bad args");
    std::vector<Layer> ly(last + 1);
    for (int j = 0; j <= last; j++) ly[j].L = layers[j];
    std::vector<int64_t> lo, hi;
    regions_1d(ly, first, last, dim, 0, b, lo, hi);
    for (int j = 0; j <= last - first; j++) ext_out[j] = hi[j] - lo[j];
    return BDL_OK;
}

// rho/tau model exposed for tests (A-2 pins).
int32_t bdl_model_brick(const bdl_plan_opts *o, int32_t nsp, int64_t N, int64_t D, int64_t H, int64_t W,
                        int64_t *rho) {
    bdl_plan_opts d;
    bdl_plan_opts_default(&d);
    int ext[4] = {(int)N, (int)D, (int)H, (int)W};
    return model_brick(o ? *o : d, nsp, ext, rho);
}

}  // extern "C"
