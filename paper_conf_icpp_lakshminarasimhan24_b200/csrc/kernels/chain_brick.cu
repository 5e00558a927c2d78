// CUDA-core merged-chain kernels at true brick granularity (one CTA works on one brick at a time).
// These execute every subgraph the tcgen05 band kernel does not cover, and the fp32 configuration
// (cfg1) whose contract is "fp32 CUDA-core path, 1e-5" (BASELINE.json north_star).
//
//   padded    (§3.2.1, Fig 2c, Fig 4): for every output brick the
//             subgraph input region of extent B + 2*sum(p) is read, then each layer is computed over
//             its (halo-padded) region into per-CTA scratch; positions outside the feature map are
//             ZERO at every intermediate layer (the next conv's zero padding).
//   memoized  (§3.2.2, Fig 2d, Fig 5): persistent CTAs draw output bricks from a
//             ticket counter and walk back through the chain with an explicit stack: for each
//             dependency brick of layer l-1, state 2 -> use; 0 -> CAS 0->1 claim, compute it first;
//             1 -> defer ("moves on ... revisits later", L523-525), then spin until 2.  Each
//             (layer, brick) is computed exactly once; a release store publishes state 2.
//   unmerged  (L659-662): one launch per layer over its output bricks.
// All modes evaluate each output element with the same fp32 accumulation order (taps outer,
// input channels inner), so padded == memoized == unmerged bit for bit.
#include <algorithm>
#include <cstring>
#include <string>

#include "common.cuh"

namespace bdl {

struct GChain {
    int L;
    int bf16;
    GLayer layer[kMaxLayers];
    TView in;
    float *scratch;
    long long slot_floats;
    int *status;
    long long task_base[kMaxLayers];
    unsigned long long *counters;   // run state (common.cuh run_epoch / run_exit)
    long long ntop;                 // bricks of the last layer's output
};

// ---- sources / destinations ------------------------------------------------------------------
template <typename T>
struct BrickSrc {
    TView v;
    __device__ __forceinline__ const T *base(int n, int d, int h, int w) const {
        return reinterpret_cast<const T *>(v.ptr) + tv_off(v, n, d, h, w);
    }
};
struct RegionBuf {  // scratch region [ext0][ext1][ext2][ext3][C] fp32
    float *p;
    int lo[4], ext[4], C;
    __device__ __forceinline__ long long idx(int n, int d, int h, int w) const {
        return ((((long long)(n - lo[0]) * ext[1] + (d - lo[1])) * ext[2] + (h - lo[2])) * ext[3] + (w - lo[3])) * C;
    }
};

__device__ __forceinline__ bool inside4(const int *e, int n, int d, int h, int w) {
    return n >= 0 && n < e[0] && d >= 0 && d < e[1] && h >= 0 && h < e[2] && w >= 0 && w < e[3];
}

// Input range [lo_in, lo_in + ext_in) of layer ly along dim i that its output range [lo, lo + ext) reads (Fig 4 reverse
// traversal): I = s(O-1) + d(k-1) + 1 for a conv / pool; a transposed conv's outputs [lo, lo+ext) gather the inputs
// i in [ceil((lo + p - d(k-1)) / s), floor((lo + ext - 1 + p) / s)].
__device__ __forceinline__ int fdiv_d(int a, int b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }
__device__ __forceinline__ void in_range(const GLayer &ly, int i, int lo, int ext, int &lo_in, int &ext_in) {
    if (ly.tr && i > 0) {
        lo_in = -fdiv_d(-(lo + ly.p[i] - ly.dl[i] * (ly.k[i] - 1)), ly.s[i]);
        ext_in = max(0, fdiv_d(lo + ext - 1 + ly.p[i], ly.s[i]) + 1 - lo_in);
    } else {
        lo_in = lo * ly.s[i] - ly.p[i];
        ext_in = (ext - 1) * ly.s[i] + ly.dl[i] * (ly.k[i] - 1) + 1;
    }
}

// Evaluate one output element (position pos, channel co) of layer `ly`.
template <typename T, bool FromRegion>
__device__ __forceinline__ float eval_elem(const GLayer &ly, const BrickSrc<T> &bs, const RegionBuf &rs,
                                           int n, int d, int h, int w, int co) {
    const bool pool = ly.kind == BDL_OP_MAXPOOL;
    float acc = pool ? -INFINITY : (ly.bias ? ly.bias[co] : 0.f);
    // grouped conv (groups = cin: depthwise): output channel co reads the cin/groups input channels of its group
    const int cin_g = ly.cin / ly.groups, c0 = pool ? 0 : (co / (ly.cout / ly.groups)) * cin_g;
    int tap = 0;
    for (int td = 0; td < ly.k[1]; td++)
        for (int th = 0; th < ly.k[2]; th++)
            for (int tw = 0; tw < ly.k[3]; tw++, tap++) {
                int id, ih, iw;
                if (ly.tr) {   // transposed conv (L378-385): input i reaches output s*i - p + d*t
                    const int nd = d + ly.p[1] - td * ly.dl[1], nh = h + ly.p[2] - th * ly.dl[2];
                    const int nw = w + ly.p[3] - tw * ly.dl[3];
                    if (nd < 0 || nh < 0 || nw < 0 || nd % ly.s[1] || nh % ly.s[2] || nw % ly.s[3]) continue;
                    id = nd / ly.s[1];
                    ih = nh / ly.s[2];
                    iw = nw / ly.s[3];
                } else {
                    id = d * ly.s[1] - ly.p[1] + td * ly.dl[1];
                    ih = h * ly.s[2] - ly.p[2] + th * ly.dl[2];
                    iw = w * ly.s[3] - ly.p[3] + tw * ly.dl[3];
                }
                if (!inside4(ly.in_ext, n, id, ih, iw)) continue;
                if (pool) {
                    float v = FromRegion ? rs.p[rs.idx(n, id, ih, iw) + co] : to_f(bs.base(n, id, ih, iw)[co]);
                    acc = fmaxf(acc, v);
                } else {
                    const float *wp = ly.w + (long long)tap * cin_g * ly.cout + co;
                    if (FromRegion) {
                        const float *xp = rs.p + rs.idx(n, id, ih, iw) + c0;
                        for (int ci = 0; ci < cin_g; ci++) acc = fmaf(wp[(long long)ci * ly.cout], xp[ci], acc);
                    } else {
                        const T *xp = bs.base(n, id, ih, iw) + c0;
                        for (int ci = 0; ci < cin_g; ci++) acc = fmaf(wp[(long long)ci * ly.cout], to_f(xp[ci]), acc);
                    }
                }
            }
    if (ly.res_ext) acc += to_f(reinterpret_cast<const T *>(ly.res.ptr)[tv_off(ly.res, n, d, h, w) + co]);
    if (ly.relu) acc = fmaxf(acc, 0.f);
    return store_round<T>(acc);
}

// Compute layer `ly` over the output region [lo, lo+ext) into either a region buffer (ToRegion) or
// the layer's bricked output view ly.out (region = exactly one brick; masked positions and padded
// channels written as 0).
template <typename T, bool FromRegion, bool ToRegion>
__device__ void layer_region(const GLayer &ly, const BrickSrc<T> &bs, const RegionBuf &rs, const RegionBuf &rd,
                             const int lo[4], const int ext[4]) {
    const int CO = ToRegion ? ly.cout : ly.out.Cp;
    long long vol = (long long)ext[0] * ext[1] * ext[2] * ext[3];
    long long total = vol * CO;
    for (long long i = threadIdx.x; i < total; i += blockDim.x) {
        int co = (int)(i % CO);
        long long pos = i / CO;
        int w = lo[3] + (int)(pos % ext[3]); pos /= ext[3];
        int h = lo[2] + (int)(pos % ext[2]); pos /= ext[2];
        int d = lo[1] + (int)(pos % ext[1]);
        int n = lo[0] + (int)(pos / ext[1]);
        float v = 0.f;
        if (co < ly.cout && inside4(ly.out_ext, n, d, h, w)) v = eval_elem<T, FromRegion>(ly, bs, rs, n, d, h, w, co);
        if (ToRegion) {
            rd.p[rd.idx(n, d, h, w) + co] = v;
        } else {
            // bricked destination: the region is a whole brick of the output grid
            T *dp = reinterpret_cast<T *>(ly.out.ptr);
            int bn = n / ly.out.B[0], bd = d / ly.out.B[1], bh = h / ly.out.B[2], bw = w / ly.out.B[3];
            long long logical = (((long long)bn * ly.out.nb[1] + bd) * ly.out.nb[2] + bh) * ly.out.nb[3] + bw;
            int inner = (((n - bn * ly.out.B[0]) * ly.out.B[1] + (d - bd * ly.out.B[1])) * ly.out.B[2] + (h - bh * ly.out.B[2])) * ly.out.B[3] + (w - bw * ly.out.B[3]);
            dp[tv_phys(ly.out, logical) * ly.out.brick_elems + (long long)inner * ly.out.Cp + co] = from_f<T>(v);
        }
    }
}

// Brick b (logical index in the grid of layer l's output) -> its origin / extent.
__device__ __forceinline__ void brick_region(const TView &o, long long b, int lo[4], int ext[4]) {
    int bw = (int)(b % o.nb[3]); b /= o.nb[3];
    int bh = (int)(b % o.nb[2]); b /= o.nb[2];
    int bd = (int)(b % o.nb[1]);
    int bn = (int)(b / o.nb[1]);
    lo[0] = bn * o.B[0]; lo[1] = bd * o.B[1]; lo[2] = bh * o.B[2]; lo[3] = bw * o.B[3];
    for (int i = 0; i < 4; i++) ext[i] = o.B[i];
}

// Compute (layer l, brick b) reading bricked input (subgraph input or memo buffer of layer l-1).
template <typename T>
__device__ void compute_brick(const GChain &g, int l, long long b) {
    const GLayer &ly = g.layer[l];
    BrickSrc<T> bs{l == 0 ? g.in : g.layer[l - 1].out};
    RegionBuf dummy{};
    int lo[4], ext[4];
    brick_region(ly.out, b, lo, ext);
    layer_region<T, false, false>(ly, bs, dummy, dummy, lo, ext);
}

// ---------------------------------------------------------------------------------------------- padded
template <typename T>
__global__ void __launch_bounds__(256) padded_chain_kernel(GChain g) {
    __shared__ int s_lo[kMaxLayers][4], s_ext[kMaxLayers][4];
    float *slot0 = g.scratch + (long long)blockIdx.x * 2 * g.slot_floats;
    float *slot1 = slot0 + g.slot_floats;
    const GLayer &last = g.layer[g.L - 1];
    for (long long t = blockIdx.x; t < g.ntop; t += gridDim.x) {
        if (threadIdx.x == 0) {
            int lo[4], ext[4];
            brick_region(last.out, t, lo, ext);
            // reverse traversal (Fig 4): output region of layer j
            for (int j = g.L - 1; j >= 0; j--) {
                for (int i = 0; i < 4; i++) { s_lo[j][i] = lo[i]; s_ext[j][i] = ext[i]; }
                const GLayer &ly = g.layer[j];
                for (int i = 0; i < 4; i++) {
                    int nlo, next;
                    in_range(ly, i, lo[i], ext[i], nlo, next);
                    lo[i] = nlo;
                    ext[i] = next;
                }
            }
        }
        __syncthreads();
        BrickSrc<T> bs{g.in};
        for (int j = 0; j < g.L; j++) {
            const GLayer &ly = g.layer[j];
            RegionBuf rs{j & 1 ? slot0 : slot1, {0}, {0}, 0};
            if (j > 0) {
                for (int i = 0; i < 4; i++) { rs.lo[i] = s_lo[j - 1][i]; rs.ext[i] = s_ext[j - 1][i]; }
                rs.C = g.layer[j - 1].cout;
            }
            RegionBuf rd{j & 1 ? slot1 : slot0, {0}, {0}, ly.cout};
            for (int i = 0; i < 4; i++) { rd.lo[i] = s_lo[j][i]; rd.ext[i] = s_ext[j][i]; }
            if (j == g.L - 1) {
                if (j == 0) layer_region<T, false, false>(ly, bs, rs, rd, rd.lo, rd.ext);
                else layer_region<T, true, false>(ly, bs, rs, rd, rd.lo, rd.ext);
            } else {
                if (j == 0) layer_region<T, false, true>(ly, bs, rs, rd, rd.lo, rd.ext);
                else layer_region<T, true, true>(ly, bs, rs, rd, rd.lo, rd.ext);
            }
            __syncthreads();
        }
        if (threadIdx.x == 0) atomicAdd(&g.counters[0], (unsigned long long)g.L);
    }
}

// ---------------------------------------------------------------------------------------------- memoized
__device__ __forceinline__ int *status_word(const GChain &g, int l, long long b) { return g.status + g.task_base[l] + b; }

// Dependencies of (l, b), l >= 1: the bricks of layer l-1's output covering layer l's input region.
struct DepBox {
    int lo[4], hi[4];  // inclusive brick index ranges
};
__device__ __forceinline__ DepBox dep_box(const GChain &g, int l, long long b) {
    const GLayer &ly = g.layer[l];
    const TView &src = g.layer[l - 1].out;
    int lo[4], ext[4];
    brick_region(ly.out, b, lo, ext);
    DepBox box;
    for (int i = 0; i < 4; i++) {
        int a, e;
        in_range(ly, i, lo[i], ext[i], a, e);
        e += a;   // exclusive
        a = max(a, 0);
        e = min(e, ly.in_ext[i]);
        box.lo[i] = a / src.B[i];
        box.hi[i] = e > a ? (e - 1) / src.B[i] : box.lo[i] - 1;
    }
    return box;
}
__device__ __forceinline__ int box_count(const DepBox &x) {
    int c = 1;
    for (int i = 0; i < 4; i++) c *= max(0, x.hi[i] - x.lo[i] + 1);
    return c;
}
__device__ __forceinline__ long long box_brick(const GChain &g, int l, const DepBox &x, int k) {
    const TView &src = g.layer[l - 1].out;
    int q[4];
    for (int i = 3; i >= 0; i--) {
        int span = x.hi[i] - x.lo[i] + 1;
        q[i] = x.lo[i] + k % span;
        k /= span;
    }
    return (((long long)q[0] * src.nb[1] + q[1]) * src.nb[2] + q[2]) * src.nb[3] + q[3];
}

struct Frame {
    int l;
    int phase;    // 0: claim pass, 1: wait pass
    int k;        // next dependency
    long long b;
};

template <typename T>
__global__ void __launch_bounds__(256) memo_chain_kernel(GChain g) {
    __shared__ Frame stk[kMaxLayers + 1];
    __shared__ int s_sp;
    __shared__ long long s_task;
    __shared__ int s_cmd_l;
    __shared__ long long s_cmd_b;
    const unsigned EP = run_epoch(g.counters) << 2;
    for (;;) {
        if (threadIdx.x == 0) {
            unsigned long long tk = atomicAdd(&g.counters[4], 1ULL);
            s_task = (long long)tk;
            if ((long long)tk < g.ntop) {
                // top-level brick: claim it (always succeeds: only tickets reach last-layer bricks)
                int *sw = status_word(g, g.L - 1, (long long)tk);
                int cur = ld_acquire(sw);  // stale epoch == state 0
                atomicCAS(sw, cur, (int)(EP | 1));
                atomicAdd(&g.counters[1], 1ULL);
                stk[0] = Frame{g.L - 1, 0, 0, (long long)tk};
                s_sp = 1;
            }
        }
        __syncthreads();
        if (s_task >= g.ntop) break;
        while (true) {
            if (threadIdx.x == 0) {
                s_cmd_l = -1;
                unsigned long long spins = 0, fails = 0, oks = 0;
                while (s_cmd_l < 0) {
                    Frame &f = stk[s_sp - 1];
                    if (f.l == 0) { s_cmd_l = 0; s_cmd_b = f.b; break; }
                    DepBox box = dep_box(g, f.l, f.b);
                    int nd = box_count(box);
                    if (f.k >= nd) {
                        if (f.phase == 0) { f.phase = 1; f.k = 0; continue; }
                        s_cmd_l = f.l; s_cmd_b = f.b;
                        break;
                    }
                    long long db = box_brick(g, f.l, box, f.k);
                    int *sw = status_word(g, f.l - 1, db);
                    int cur = ld_acquire(sw);
                    bool fresh = (cur & ~3) == (int)EP;
                    int st = fresh ? (cur & 3) : 0;
                    if (f.phase == 0) {
                        f.k++;
                        if (st == 2) continue;
                        if (st == 0) {
                            int prev = atomicCAS(sw, cur, (int)(EP | 1));
                            if (prev == cur) {
                                oks++;
                                stk[s_sp] = Frame{f.l - 1, 0, 0, db};
                                s_sp++;
                                continue;
                            }
                        }
                        fails++;  // in progress elsewhere: revisit in the wait pass
                    } else {
                        if (st == 2) { f.k++; continue; }
                        spins++;
                        __nanosleep(64);
                    }
                }
                if (oks) atomicAdd(&g.counters[1], oks);
                if (fails) atomicAdd(&g.counters[2], fails);
                if (spins) atomicAdd(&g.counters[3], spins);
                __threadfence();
            }
            __syncthreads();
            int l = s_cmd_l;
            long long b = s_cmd_b;
            compute_brick<T>(g, l, b);
            __syncthreads();
            if (threadIdx.x == 0) {
                __threadfence();
                st_release(status_word(g, l, b), (int)(EP | 2));
                atomicAdd(&g.counters[0], 1ULL);
                s_sp--;
            }
            __syncthreads();
            if (s_sp == 0) break;
        }
    }
    if (threadIdx.x == 0) run_exit(g.counters);
}

// ---------------------------------------------------------------------------------------------- unmerged
template <typename T>
__global__ void __launch_bounds__(256) layer_kernel(GChain g, int l) {
    long long nb = (long long)g.layer[l].out.nb[0] * g.layer[l].out.nb[1] * g.layer[l].out.nb[2] * g.layer[l].out.nb[3];
    for (long long b = blockIdx.x; b < nb; b += gridDim.x) {
        compute_brick<T>(g, l, b);
        __syncthreads();
    }
    if (threadIdx.x == 0 && blockIdx.x == 0) atomicAdd(&g.counters[0], (unsigned long long)nb);
}

// Max-pool (L456-458; out-of-range taps ignored) as its own HBM-bound layer kernel: one
// thread per (output pixel, 16-byte channel vector), 16-B loads of each in-range window tap and one
// 16-B store into the bricked output (consecutive threads -> consecutive 16-B chunks of a brick, so
// loads and stores are coalesced along the channels-innermost brick rows).  Masked positions of
// partial bricks and padded channels are written as 0 (Q11).
// Element offset of channel 0 at (n, d, h, w) for power-of-two brick extents (log2 in lB[0..3]).
__device__ __forceinline__ long long tv_off_p2(const TView &v, const int *lB, int n, int d, int h, int w) {
    const int bn = n >> lB[0], bd = d >> lB[1], bh = h >> lB[2], bw = w >> lB[3];
    const long long logical = (((long long)bn * v.nb[1] + bd) * v.nb[2] + bh) * v.nb[3] + bw;
    const int in = ((((((n - (bn << lB[0])) << lB[1]) + (d - (bd << lB[1]))) << lB[2]) + (h - (bh << lB[2])))
                    << lB[3]) + (w - (bw << lB[3]));
    return tv_phys(v, logical) * v.brick_elems + (long long)in * v.Cp;
}

// K > 0: a 2-D K x K window, unrolled so that all its loads are in flight at once (the generic loop waits for each tap's
// load before the next: ~3 TB/s on VGG-16's pools)
template <typename T, bool P2, int K>
__global__ void __launch_bounds__(256) pool_vec_kernel(GLayer ly, TView in, unsigned long long *counter, int4 lb4) {
    const int lB[4] = {lb4.x, lb4.y, lb4.z, lb4.w};
    constexpr int V = 16 / sizeof(T);
    const TView &o = ly.out;
    const int nvec = o.Cp / V;
    const int bpx = o.B[0] * o.B[1] * o.B[2] * o.B[3];
    const long long nbr = (long long)o.nb[0] * o.nb[1] * o.nb[2] * o.nb[3];
    const long long total = nbr * bpx * nvec;
    int lnv = 0, lbpx = lB[0] + lB[1] + lB[2] + lB[3];
    while ((1 << lnv) < nvec) lnv++;
    if ((1 << lnv) != nvec) lnv = -1;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
        int cv, inner, inner0;
        long long b;   // logical brick
        if (P2 && lnv >= 0) {   // shifts only (power-of-two vectors per pixel and pixels per brick)
            cv = (int)(i & (nvec - 1));
            const long long r = i >> lnv;
            inner = (int)(r & (bpx - 1));
            b = r >> lbpx;
        } else {
            cv = (int)(i % nvec);
            const long long r = i / nvec;
            inner = (int)(r % bpx);
            b = r / bpx;
        }
        inner0 = inner;
        int lo[4], ext[4];
        brick_region(o, b, lo, ext);
        int w, h, d, n;
        if (P2) {
            w = lo[3] + (inner & ((1 << lB[3]) - 1)); inner >>= lB[3];
            h = lo[2] + (inner & ((1 << lB[2]) - 1)); inner >>= lB[2];
            d = lo[1] + (inner & ((1 << lB[1]) - 1));
            n = lo[0] + (inner >> lB[1]);
        } else {
            w = lo[3] + inner % o.B[3]; inner /= o.B[3];
            h = lo[2] + inner % o.B[2]; inner /= o.B[2];
            d = lo[1] + inner % o.B[1];
            n = lo[0] + inner / o.B[1];
        }
        float m[V];
#pragma unroll
        for (int j = 0; j < V; j++) m[j] = -INFINITY;
        bool any = false;
        if (K > 0 && inside4(ly.out_ext, n, d, h, w)) {
            constexpr int KK = K > 0 ? K * K : 1;
            uint4 q[KK];
            bool ok[KK];
#pragma unroll
            for (int th = 0; th < K; th++)
#pragma unroll
                for (int tw = 0; tw < K; tw++) {
                    const int ih = h * ly.s[2] - ly.p[2] + th, iw = w * ly.s[3] - ly.p[3] + tw;
                    const int id = d * ly.s[1] - ly.p[1];
                    ok[th * K + tw] = inside4(ly.in_ext, n, id, ih, iw);
                    const long long eo = ok[th * K + tw] ? (P2 ? tv_off_p2(in, lB, n, id, ih, iw) : tv_off(in, n, id, ih, iw)) : 0;
                    q[th * K + tw] = __ldg(reinterpret_cast<const uint4 *>(reinterpret_cast<const T *>(in.ptr) + eo + cv * V));
                }
#pragma unroll
            for (int t = 0; t < K * K; t++) {
                if (!ok[t]) continue;
                const T *e = reinterpret_cast<const T *>(&q[t]);
#pragma unroll
                for (int j = 0; j < V; j++) m[j] = fmaxf(m[j], to_f(e[j]));
                any = true;
            }
        } else if (K == 0 && inside4(ly.out_ext, n, d, h, w)) {
            for (int td = 0; td < ly.k[1]; td++) {
                const int id = d * ly.s[1] - ly.p[1] + td;
                for (int th = 0; th < ly.k[2]; th++) {
                    const int ih = h * ly.s[2] - ly.p[2] + th;
                    for (int tw = 0; tw < ly.k[3]; tw++) {
                        const int iw = w * ly.s[3] - ly.p[3] + tw;
                        if (!inside4(ly.in_ext, n, id, ih, iw)) continue;
                        const long long eo = P2 ? tv_off_p2(in, lB, n, id, ih, iw) : tv_off(in, n, id, ih, iw);
                        const uint4 q = __ldg(reinterpret_cast<const uint4 *>(reinterpret_cast<const T *>(in.ptr) + eo + cv * V));
                        const T *e = reinterpret_cast<const T *>(&q);
#pragma unroll
                        for (int j = 0; j < V; j++) m[j] = fmaxf(m[j], to_f(e[j]));
                        any = true;
                    }
                }
            }
        }
        uint4 outv;
        T *oe = reinterpret_cast<T *>(&outv);
#pragma unroll
        for (int j = 0; j < V; j++) {
            float v = (any && cv * V + j < ly.cout) ? m[j] : 0.f;
            if (ly.relu) v = fmaxf(v, 0.f);
            oe[j] = from_f<T>(v);
        }
        *reinterpret_cast<uint4 *>(reinterpret_cast<T *>(o.ptr) + tv_phys(o, b) * o.brick_elems +
                                   (long long)inner0 * o.Cp + cv * V) = outv;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(counter, (unsigned long long)nbr);
}

// weights [cout][kd][kh][kw][cin] (dtype) -> [taps][cin][cout] fp32
template <typename T>
__global__ void pack_weights_f32_kernel(const T *__restrict__ w, float *__restrict__ out, int cout, int taps, int cin,
                                        const float *__restrict__ bias, float *__restrict__ bout) {
    long long total = (long long)cout * taps * cin;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
        int ci = (int)(i % cin);
        long long r = i / cin;
        int t = (int)(r % taps);
        int co = (int)(r / taps);
        out[((long long)t * cin + ci) * cout + co] = to_f(w[i]);
    }
    if (blockIdx.x == 0)
        for (int co = threadIdx.x; co < cout; co += blockDim.x) bout[co] = bias ? bias[co] : 0.f;
}

// ---------------------------------------------------------------------------------------------- host
bdl_status launch_pack_f32(const bdl_layer &l, int dtype, float *w_out, float *b_out, cudaStream_t s) {
    int taps = l.k[0] * l.k[1] * l.k[2];
    const int cin_g = l.cin / (l.groups > 1 ? l.groups : 1);   // grouped weights [cout][taps][cin/groups]
    long long total = (long long)l.cout * taps * cin_g;
    int grid = (int)std::min<long long>((total + 255) / 256, 4096);
    if (dtype == BDL_F32)
        pack_weights_f32_kernel<float><<<grid, 256, 0, s>>>((const float *)l.w, w_out, l.cout, taps, cin_g, l.bias, b_out);
    else
        pack_weights_f32_kernel<__nv_bfloat16><<<grid, 256, 0, s>>>((const __nv_bfloat16 *)l.w, w_out, l.cout, taps, cin_g, l.bias, b_out);
    BDL_CUDA_CHECK_LAUNCH("pack_weights");
    return BDL_OK;
}

// Build the device descriptor of subgraph `sg` and launch its CUDA-core kernel(s).
bdl_status launch_brick_subgraph(bdl_plan *p, const Subgraph &sg, const TView &in, const TView &out,
                                 const std::vector<TView> &res_views, unsigned char *ws, cudaStream_t s,
                                 int *launches) {
    GChain g;
    memset(&g, 0, sizeof(g));
    g.L = sg.last - sg.first + 1;
    g.bf16 = p->in_layout.dtype == BDL_BF16;
    g.in = in;
    for (int j = 0; j < g.L; j++) {
        const Layer &ly = p->layers[sg.first + j];
        GLayer &G = g.layer[j];
        G.kind = ly.L.kind;
        G.cin = ly.L.cin;
        G.cout = ly.L.cout;
        G.k[0] = 1; G.s[0] = 1; G.p[0] = 0; G.dl[0] = 1;
        for (int d = 0; d < 3; d++) {
            G.k[d + 1] = ly.L.k[d]; G.s[d + 1] = ly.L.stride[d]; G.p[d + 1] = ly.L.pad[d]; G.dl[d + 1] = ly.L.dil[d];
        }
        G.groups = ly.L.groups;
        G.tr = ly.L.transposed;
        for (int d = 0; d < 4; d++) { G.in_ext[d] = ly.in_ext[d]; G.out_ext[d] = ly.out_ext[d]; }
        G.relu = ly.L.relu;
        G.w = ly.L.kind == BDL_OP_CONV ? (const float *)(ws + ly.w_off) : nullptr;
        G.bias = ly.L.kind == BDL_OP_CONV ? (const float *)(ws + ly.b_off) : nullptr;
        G.res_ext = sg.res_tensor[j] >= 0;
        if (G.res_ext) G.res = res_views[j];
        if (j == g.L - 1) {
            G.out = out;
        } else {
            bdl_layout lo;
            bdl_layout_init(&lo, p->in_layout.nsp, ly.out_ext[0], ly.L.cout, ly.out_ext[1], ly.out_ext[2], ly.out_ext[3],
                            p->in_layout.Bn, p->in_layout.Bd, p->in_layout.Bh, p->in_layout.Bw, p->in_layout.dtype);
            G.out = make_view(lo, ws + sg.memo_off[j]);
        }
    }
    const TView &o = g.layer[g.L - 1].out;
    g.ntop = (long long)o.nb[0] * o.nb[1] * o.nb[2] * o.nb[3];
    g.scratch = sg.scratch_off >= 0 ? (float *)(ws + sg.scratch_off) : nullptr;
    g.slot_floats = sg.scratch_slot_floats;
    g.status = (int *)(ws + sg.status_off);
    for (int j = 0; j < g.L; j++) g.task_base[j] = sg.task_base[j];
    g.counters = (unsigned long long *)(ws + sg.counter_off);
    int grid = (int)std::min<long long>(g.ntop, sg.grid);
    int mode = sg.mode;
    if (g.L == 1) mode = BDL_MODE_UNMERGED;
    if (mode == BDL_MODE_PADDED) {
        if (g.bf16) padded_chain_kernel<__nv_bfloat16><<<grid, 256, 0, s>>>(g);
        else padded_chain_kernel<float><<<grid, 256, 0, s>>>(g);
        *launches += 1;
    } else if (mode == BDL_MODE_MEMOIZED) {
        if (g.bf16) memo_chain_kernel<__nv_bfloat16><<<grid, 256, 0, s>>>(g);
        else memo_chain_kernel<float><<<grid, 256, 0, s>>>(g);
        *launches += 1;
    } else {
        for (int l = 0; l < g.L; l++) {
            const TView &ov = g.layer[l].out;
            long long nb = (long long)ov.nb[0] * ov.nb[1] * ov.nb[2] * ov.nb[3];
            const GLayer &G = g.layer[l];
            const int esz = g.bf16 ? 2 : 4;
            const TView &src = l == 0 ? g.in : g.layer[l - 1].out;
            if (G.kind == BDL_OP_MAXPOOL && !G.res_ext && (G.out.Cp * esz) % 16 == 0 && (src.Cp * esz) % 16 == 0) {
                const long long threads = nb * G.out.B[0] * G.out.B[1] * G.out.B[2] * G.out.B[3] * (G.out.Cp * esz / 16);
                const int gp = (int)std::min<long long>((threads + 255) / 256, 148LL * 64);
                auto lg = [](int v) { int r = 0; while ((1 << r) < v) r++; return (1 << r) == v ? r : -1; };
                const int4 lb4 = make_int4(lg(src.B[0]), lg(src.B[1]), lg(src.B[2]), lg(src.B[3]));
                const bool p2 = lb4.x >= 0 && lb4.y >= 0 && lb4.z >= 0 && lb4.w >= 0;
                const int kk = G.k[1] == 1 && G.k[2] == G.k[3] && (G.k[2] == 2 || G.k[2] == 3) ? G.k[2] : 0;
#define BDL_POOL_LAUNCH(TT, PP)                                                                            \
    do {                                                                                                  \
        if (kk == 2) pool_vec_kernel<TT, PP, 2><<<gp, 256, 0, s>>>(G, src, g.counters, lb4);              \
        else if (kk == 3) pool_vec_kernel<TT, PP, 3><<<gp, 256, 0, s>>>(G, src, g.counters, lb4);         \
        else pool_vec_kernel<TT, PP, 0><<<gp, 256, 0, s>>>(G, src, g.counters, lb4);                       \
    } while (0)
                if (g.bf16) {
                    if (p2) BDL_POOL_LAUNCH(__nv_bfloat16, true);
                    else BDL_POOL_LAUNCH(__nv_bfloat16, false);
                } else {
                    if (p2) BDL_POOL_LAUNCH(float, true);
                    else BDL_POOL_LAUNCH(float, false);
                }
#undef BDL_POOL_LAUNCH
                *launches += 1;
                continue;
            }
            int gl = (int)std::min<long long>(nb, 65535LL * 16);
            if (g.bf16) layer_kernel<__nv_bfloat16><<<gl, 256, 0, s>>>(g, l);
            else layer_kernel<float><<<gl, 256, 0, s>>>(g, l);
            *launches += 1;
        }
    }
    BDL_CUDA_CHECK_LAUNCH("brick chain kernel");
    return BDL_OK;
}

}  // namespace bdl
