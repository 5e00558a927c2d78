// tcgen05 band kernels: merged 3x3 conv chains in bf16 on the 5th-generation tensor cores.
//
// Implicit-GEMM formulation (one layer, one output tile of Tb rows x Tw columns, C channels):
//   The input tile (Tb + 2 halo rows) x Wt columns (Wt = Tw + 2*halo) is staged in shared memory as
//   C/8 "chunk planes", each [rows][16 B] (8 bf16 channels per 16-byte row).  That is exactly the
//   UMMA K-major SWIZZLE_NONE canonical layout with SBO = 128 B (8 consecutive pixels) and
//   LBO = chunk-plane stride, so the A operand of tap (r, s) is the same buffer with its start
//   address advanced by (r*Wt + s) pixels: out[m] = sum_{r,s} W_rs * in[m + r*Wt + s] for the
//   flattened pixel index m = i*Wt + j.  Columns j >= Tw are computed and discarded.
//   M = 128 pixels per MMA, N = C output channels, K = 16 input channels; accumulators live in TMEM
//   (one 128 x C fp32 block per M tile); weights stream tap by tap through a 3-stage shared-memory
//   ring filled by the TMA engine (cp.async.bulk) and released by tcgen05.commit.
//
// Modes (§3.2):
//   padded   (§3.2.1, Fig 4): one CTA computes all L layers of an output tile; layer j's output
//            (region shrinking by one pixel per side per layer) stays in shared memory as the next
//            layer's A operand; positions outside the feature map are written as ZERO.
//   memoized (§3.2.2, Fig 5): a task is one (layer, image, tile).  Persistent CTAs draw output tiles
//            from a ticket counter and walk back with the three-state CAS protocol of chain_brick.cu;
//            intermediate tiles are published to bricked global (L2-resident) buffers.
//   unmerged : one launch per layer over all tiles (the memo kernel with dependency checks off).
// Epilogue order: + bias -> + residual -> ReLU -> bf16 RNE.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "common.cuh"
#include "tc_ptx.cuh"

namespace bdl {

static unsigned long long *trace_buf = nullptr;  // debug task trace (BDL_TRACE=<capacity>)

constexpr int kNS = 3;          // weight ring stages (one tap each)
constexpr int kTcThreads = 128; // 4 warps: warp w owns TMEM lanes [32w, 32w+32)

struct TcLayer {
    const __nv_bfloat16 *w;  // packed [9][C/8][C][8]
    const float *bias;
    int relu;
    int res;                 // add the residual view at this layer
    TView out;
};

struct TcParams {
    int mode;
    int L, C;
    int N, H, W;
    int Tb, Tw, Wt;
    int nty, ntx;
    int rowsA, rowsB;
    int tmem_cols;
    TcLayer layer[kMaxLayers];
    TView in, res;
    int *status;
    long long task_base[kMaxLayers];
    unsigned long long *counters;  // [0] tiles computed (common.cuh counter block)
    long long ntiles;              // tiles per layer = N * nty * ntx
    int only_layer;                // >= 0: unmerged launch of that layer
    unsigned long long *trace;     // debug: per task [smid|l, tile, t0..t4] (globaltimer ns), or null
    int trace_cap;
};

__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned smid() {
    unsigned r;
    asm volatile("mov.u32 %0, %smid;" : "=r"(r));
    return r;
}

struct TcShared {   // static shared state
    uint64_t full[kNS], empty[kNS], mma_done;
    uint32_t tmem_base;
    int cmd_l, sp;
    long long cmd_t, task;
};

// ------------------------------------------------------------------------------------------------
// Stage a tile of `src` (bricked, bf16) into chunk planes: pixel q = a*Wt + b <-> image
// (y_org + a, x_org + b), rows a in [0, R).  Outside the image -> zero (cp.async zero-fill).
template <int C>
__device__ __forceinline__ void load_tile(const TView &src, int n, int y_org, int x_org, int R, int Wt,
                                          uint8_t *buf, int rows_alloc) {
    constexpr int KC = C / 8;
    const __nv_bfloat16 *base = reinterpret_cast<const __nv_bfloat16 *>(src.ptr);
    const int items = R * Wt * KC;
    for (int i = threadIdx.x; i < items; i += kTcThreads) {
        int k = i % KC;
        int q = i / KC;
        int a = q / Wt;
        int y = y_org + a, x = x_org + (q - a * Wt);
        bool ok = y >= 0 && y < src.ext[2] && x >= 0 && x < src.ext[3];
        const void *g = ok ? (const void *)(base + tv_off(src, n, 0, y, x) + k * 8) : (const void *)base;
        ptx::cp_async16(buf + ((size_t)k * rows_alloc + q) * 16, g, ok ? 16u : 0u);
    }
    ptx::cp_async_wait_all();
    ptx::fence_proxy_async_smem();
}

// One layer of MMAs over `ntiles` M-tiles of the A buffer; single issuing thread.
template <int C>
__device__ __forceinline__ void issue_layer(const TcParams &p, TcShared &sh, const __nv_bfloat16 *w, const uint8_t *abuf,
                                            int rows_alloc, int ntiles, uint8_t *wst, uint32_t &wq) {
    constexpr uint32_t WB = C * C * 2;
    constexpr uint32_t LBO_B = C * 16;
    constexpr uint32_t IDESC = ptx::idesc_bf16_f32(128, C);
    const uint32_t LBO_A = (uint32_t)rows_alloc * 16;
    const uint32_t a_base = ptx::smem_u32(abuf);
    const uint32_t w_base = ptx::smem_u32(wst);
    auto issue = [&](int tap) {
        uint32_t g = wq + tap;
        int st = g % kNS;
        uint32_t use = g / kNS;
        if (use > 0) ptx::mbar_wait(&sh.empty[st], (use - 1) & 1);
        ptx::mbar_arrive_expect_tx(&sh.full[st], WB);
        ptx::bulk_g2s(wst + st * WB, w + (size_t)tap * C * C, WB, &sh.full[st]);
    };
    for (int t = 0; t < kNS; t++) issue(t);
    for (int tap = 0; tap < 9; tap++) {
        uint32_t g = wq + tap;
        int st = g % kNS;
        ptx::mbar_wait(&sh.full[st], (g / kNS) & 1);
        ptx::tc_fence_after();
        const int shift = (tap / 3) * p.Wt + (tap % 3);
        const uint32_t b0 = w_base + st * WB;
        for (int t = 0; t < ntiles; t++) {
            const uint32_t arow = a_base + (uint32_t)(t * 128 + shift) * 16;
#pragma unroll
            for (int kk = 0; kk < C / 16; kk++) {
                uint64_t ad = ptx::umma_desc_noswz(arow + 2 * kk * LBO_A, LBO_A, 128);
                uint64_t bd = ptx::umma_desc_noswz(b0 + 2 * kk * LBO_B, LBO_B, 128);
                ptx::mma_bf16(sh.tmem_base + t * C, ad, bd, IDESC, (tap | kk) != 0);
            }
        }
        ptx::mma_commit(&sh.empty[st]);
        if (tap >= 1 && tap - 1 + kNS < 9) issue(tap - 1 + kNS);
    }
    wq += 9;
    ptx::mma_commit(&sh.mma_done);
}

__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
    __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<uint32_t *>(&v);
}

// Epilogue to global bricked output: tile origin (n, y0, x0), rows m -> (m / Wt, m % Wt).
template <int C>
__device__ __forceinline__ void epilogue_global(const TcParams &p, TcShared &sh, const TcLayer &ly, int ntiles, int n,
                                                int y0, int x0, bool add_res) {
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    __nv_bfloat16 *outp = reinterpret_cast<__nv_bfloat16 *>(ly.out.ptr);
    const __nv_bfloat16 *resp = reinterpret_cast<const __nv_bfloat16 *>(p.res.ptr);
    for (int t = 0; t < ntiles; t++) {
        uint32_t r[C / 16][16];
        const uint32_t taddr = sh.tmem_base + ((uint32_t)(warp * 32) << 16) + t * C;
#pragma unroll
        for (int cc = 0; cc < C / 16; cc++) ptx::tmem_ld16(taddr + cc * 16, r[cc]);
        ptx::tmem_ld_wait();
        int m = t * 128 + warp * 32 + lane;
        int i = m / p.Wt, j = m - (m / p.Wt) * p.Wt;
        if (i >= p.Tb || j >= p.Tw) continue;
        int y = y0 + i, x = x0 + j;
        if (y >= ly.out.ext[2] || x >= ly.out.ext[3]) {
            if (y < ly.out.nb[2] * ly.out.B[2] && x < ly.out.nb[3] * ly.out.B[3]) {  // masked part of a brick
                uint4 *dst = reinterpret_cast<uint4 *>(outp + tv_off(ly.out, n, 0, y, x));
#pragma unroll
                for (int k = 0; k < C / 8; k++) dst[k] = make_uint4(0, 0, 0, 0);
            }
            continue;
        }
        uint4 *dst = reinterpret_cast<uint4 *>(outp + tv_off(ly.out, n, 0, y, x));
        const uint4 *rs = add_res ? reinterpret_cast<const uint4 *>(resp + tv_off(p.res, n, 0, y, x)) : nullptr;
#pragma unroll
        for (int k = 0; k < C / 8; k++) {
            float v[8];
#pragma unroll
            for (int e = 0; e < 8; e++) v[e] = __uint_as_float(r[k / 2][(k % 2) * 8 + e]) + ly.bias[k * 8 + e];
            if (add_res) {
                uint4 rv = __ldcg(rs + k);
                const __nv_bfloat162 *h = reinterpret_cast<const __nv_bfloat162 *>(&rv);
#pragma unroll
                for (int e = 0; e < 4; e++) {
                    float2 f = __bfloat1622float2(h[e]);
                    v[2 * e] += f.x;
                    v[2 * e + 1] += f.y;
                }
            }
            if (ly.relu) {
#pragma unroll
                for (int e = 0; e < 8; e++) v[e] = fmaxf(v[e], 0.f);
            }
            dst[k] = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                                pack_bf16x2(v[6], v[7]));
        }
    }
}

// Epilogue to a shared-memory chunk-plane buffer (padded mode intermediate): rows m < Mrows;
// pixel (m / Wt, m % Wt) <-> image (yo + i, xo + j); valid columns j < vcols; outside -> 0.
template <int C>
__device__ __forceinline__ void epilogue_smem(const TcParams &p, TcShared &sh, const TcLayer &ly, int ntiles, int Mrows,
                                              int yo, int xo, int vcols, uint8_t *dbuf, int rows_alloc) {
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    for (int t = 0; t < ntiles; t++) {
        uint32_t r[C / 16][16];
        const uint32_t taddr = sh.tmem_base + ((uint32_t)(warp * 32) << 16) + t * C;
#pragma unroll
        for (int cc = 0; cc < C / 16; cc++) ptx::tmem_ld16(taddr + cc * 16, r[cc]);
        ptx::tmem_ld_wait();
        int m = t * 128 + warp * 32 + lane;
        if (m >= Mrows) continue;
        int i = m / p.Wt, j = m - (m / p.Wt) * p.Wt;
        int y = yo + i, x = xo + j;
        bool valid = j < vcols && y >= 0 && y < p.H && x >= 0 && x < p.W;
#pragma unroll
        for (int k = 0; k < C / 8; k++) {
            uint4 o = make_uint4(0, 0, 0, 0);
            if (valid) {
                float v[8];
#pragma unroll
                for (int e = 0; e < 8; e++) {
                    v[e] = __uint_as_float(r[k / 2][(k % 2) * 8 + e]) + ly.bias[k * 8 + e];
                    if (ly.relu) v[e] = fmaxf(v[e], 0.f);
                }
                o = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                               pack_bf16x2(v[6], v[7]));
            }
            *reinterpret_cast<uint4 *>(dbuf + ((size_t)k * rows_alloc + m) * 16) = o;
        }
    }
    ptx::fence_proxy_async_smem();
}

__device__ __forceinline__ void decode_tile(const TcParams &p, long long t, int &n, int &ty, int &tx) {
    tx = (int)(t % p.ntx);
    t /= p.ntx;
    ty = (int)(t % p.nty);
    n = (int)(t / p.nty);
}

template <int C>
__device__ __forceinline__ void setup(TcShared &sh, uint8_t *smem, int zero_bytes, int tmem_cols) {
    if (threadIdx.x == 0) {
        for (int i = 0; i < kNS; i++) {
            ptx::mbar_init(&sh.full[i], 1);
            ptx::mbar_init(&sh.empty[i], 1);
        }
        ptx::mbar_init(&sh.mma_done, 1);
        ptx::fence_barrier_init();
    }
    if (threadIdx.x / 32 == 0) {
        ptx::tmem_alloc(&sh.tmem_base, tmem_cols);
        ptx::tmem_relinquish();
    }
    // zero the activation buffers once: guard rows are never written by the loader
    for (int i = threadIdx.x * 16; i < zero_bytes; i += kTcThreads * 16)
        *reinterpret_cast<uint4 *>(smem + i) = make_uint4(0, 0, 0, 0);
    ptx::fence_proxy_async_smem();
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
}

template <int C>
__device__ __forceinline__ void teardown(TcShared &sh, int tmem_cols) {
    ptx::tc_fence_before();
    __syncthreads();
    if (threadIdx.x / 32 == 0) ptx::tmem_dealloc(sh.tmem_base, tmem_cols);
}

// ------------------------------------------------------------------------------------------------ padded
template <int C>
__global__ void __launch_bounds__(kTcThreads, 1) tc_padded_kernel(const __grid_constant__ TcParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ TcShared sh;
    constexpr int KC = C / 8;
    uint8_t *bufA = smem;
    uint8_t *bufB = bufA + (size_t)KC * p.rowsA * 16;
    uint8_t *wst = bufB + (size_t)KC * p.rowsB * 16;
    setup<C>(sh, smem, KC * (p.rowsA + p.rowsB) * 16, p.tmem_cols);
    uint32_t wq = 0, done_phase = 0;
    const int L = p.L;
    for (long long t = blockIdx.x; t < p.ntiles; t += gridDim.x) {
        int n, ty, tx;
        decode_tile(p, t, n, ty, tx);
        const int y0 = ty * p.Tb, x0 = tx * p.Tw;
        load_tile<C>(p.in, n, y0 - L, x0 - L, p.Tb + 2 * L, p.Wt, bufA, p.rowsA);
        __syncthreads();
        for (int j = 0; j < L; j++) {
            uint8_t *src = (j & 1) ? bufB : bufA;
            uint8_t *dst = (j & 1) ? bufA : bufB;
            int src_rows = (j & 1) ? p.rowsB : p.rowsA, dst_rows = (j & 1) ? p.rowsA : p.rowsB;
            const int Mrows = (p.Tb + 2 * (L - 1 - j)) * p.Wt;
            const int ntl = (Mrows + 127) / 128;
            ptx::tc_fence_after();
            if (threadIdx.x == 0) issue_layer<C>(p, sh, p.layer[j].w, src, src_rows, ntl, wst, wq);
            ptx::mbar_wait(&sh.mma_done, done_phase);
            done_phase ^= 1;
            ptx::tc_fence_after();
            if (j == L - 1) {
                epilogue_global<C>(p, sh, p.layer[j], ntl, n, y0, x0, p.layer[j].res);
            } else {
                const int off = L - 1 - j;  // output origin relative to the tile origin
                epilogue_smem<C>(p, sh, p.layer[j], ntl, Mrows, y0 - off, x0 - off, p.Wt - 2 * (j + 1), dst, dst_rows);
            }
            ptx::tc_fence_before();
            __syncthreads();
        }
        if (threadIdx.x == 0) atomicAdd(&p.counters[0], (unsigned long long)L);
    }
    teardown<C>(sh, p.tmem_cols);
}

// weights [cout][3][3][cin] (bf16) -> [tap][cin/8][cout][8]
__global__ void pack_tc_kernel(const __nv_bfloat16 *__restrict__ w, __nv_bfloat16 *__restrict__ out, int C, int taps) {
    long long total = (long long)C * taps * C;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
        int ci = (int)(i % C);
        long long r = i / C;
        int t = (int)(r % taps);
        int co = (int)(r / taps);
        out[(((long long)t * (C / 8) + ci / 8) * C + co) * 8 + (ci % 8)] = w[i];
    }
}

// ------------------------------------------------------------------------------------------------ host
struct TcGeom {
    int Tb, Tw, Wt, rowsA, rowsB, smem, tmem_cols, ntl_max;
};

static int round_rows(int r) { return (r + 7) / 8 * 8 + 1; }  // odd multiple of 16 B: conflict-free stores

static bool tc_geometry(const bdl_plan *p, const Subgraph &sg, int mode, TcGeom &g) {
    const Layer &f = p->layers[sg.first];
    const int C = f.L.cin;
    const int L = sg.last - sg.first + 1;
    const int H = f.in_ext[2], W = f.in_ext[3];
    const int Bh = p->in_layout.Bh, Bw = p->in_layout.Bw;
    if (p->in_layout.nsp != 2) return false;
    const int wbytes = kNS * C * C * 2;
    const int limit = 227 * 1024 - 1024;
    int Wfull = (W + Bw - 1) / Bw * Bw;
    for (int Tw = Wfull; Tw >= Bw; Tw -= Bw) {
        g.Tb = Bh;
        g.Tw = Tw;
        if (mode == BDL_MODE_PADDED) {
            g.Wt = Tw + 2 * L;
            int M0 = (g.Tb + 2 * (L - 1)) * g.Wt;
            int n0 = (M0 + 127) / 128;
            g.rowsA = round_rows(n0 * 128 + 2 * g.Wt + 2);
            int M1 = L > 1 ? (g.Tb + 2 * (L - 2)) * g.Wt : 0;
            int n1 = (M1 + 127) / 128;
            g.rowsB = L > 1 ? round_rows(std::max(M0, n1 * 128 + 2 * g.Wt + 2)) : 0;
            g.ntl_max = n0;
        } else {
            g.Wt = Tw + 2;
            int M = g.Tb * g.Wt;
            int n0 = (M + 127) / 128;
            g.rowsA = round_rows(n0 * 128 + 2 * g.Wt + 2);
            g.rowsB = 0;
            g.ntl_max = n0;
        }
        g.smem = (C / 8) * (g.rowsA + g.rowsB) * 16 + wbytes;
        int cols = g.ntl_max * C;
        g.tmem_cols = 32;
        while (g.tmem_cols < cols) g.tmem_cols *= 2;
        if (g.smem <= limit && cols <= 512) return true;
    }
    (void)H;
    return false;
}

int tc_band_rows(const bdl_plan *p, const Subgraph &sg, int *smem_out) {
    TcGeom a, b;
    bool okm = tc_geometry(p, sg, BDL_MODE_MEMOIZED, a);
    bool okp = (sg.last == sg.first) || tc_geometry(p, sg, BDL_MODE_PADDED, b);
    if (!okm || !okp) return 0;
    *smem_out = a.smem;
    return a.Tb;
}

int tc_launches(const bdl_plan *p, const Subgraph &sg) {
    int L = sg.last - sg.first + 1;
    return (sg.mode == BDL_MODE_UNMERGED || L == 1) ? L : 1;
}

bdl_status launch_pack_tc(const bdl_layer &l, void *w_out, cudaStream_t s) {
    int taps = l.k[0] * l.k[1] * l.k[2];
    long long total = (long long)l.cout * taps * l.cin;
    int grid = (int)std::min<long long>((total + 255) / 256, 4096);
    pack_tc_kernel<<<grid, 256, 0, s>>>((const __nv_bfloat16 *)l.w, (__nv_bfloat16 *)w_out, l.cin, taps);
    BDL_CUDA_CHECK_LAUNCH("pack_tc");
    return BDL_OK;
}

template <int C>
static bdl_status launch_tc_C(bdl_plan *p, Subgraph &sg, TcParams &P, const TcGeom &g, int mode, cudaStream_t s,
                              int *launches) {
    const int ctas_per_sm = g.smem <= 113 * 1024 ? 2 : 1;
    if (mode == BDL_MODE_PADDED) {
        auto k = tc_padded_kernel<C>;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, g.smem);
        int grid = (int)std::min<long long>(P.ntiles, (long long)p->num_sms * ctas_per_sm);
        k<<<grid, kTcThreads, g.smem, s>>>(P);
        *launches += 1;
    } else {
        return fail(BDL_EUNSUPPORTED, "tc band kernel: memoized / unmerged modes run on the warp-specialized kernel");
    }
    BDL_CUDA_CHECK_LAUNCH("tc chain kernel");
    return BDL_OK;
}

bdl_status launch_tc_subgraph(bdl_plan *p, Subgraph &sg, const TView &in, const TView &out, const TView *res,
                              unsigned char *ws, cudaStream_t s, int *launches) {
    int L = sg.last - sg.first + 1;
    int mode = L == 1 ? BDL_MODE_UNMERGED : sg.mode;
    TcGeom g;
    if (!tc_geometry(p, sg, mode == BDL_MODE_PADDED ? BDL_MODE_PADDED : BDL_MODE_MEMOIZED, g))
        return fail(BDL_EUNSUPPORTED, "tcgen05 band kernel: tile does not fit on chip");
    TcParams P;
    memset(&P, 0, sizeof(P));
    const Layer &f = p->layers[sg.first];
    P.mode = mode;
    P.L = L;
    P.C = f.L.cin;
    P.N = f.in_ext[0];
    P.H = f.in_ext[2];
    P.W = f.in_ext[3];
    P.Tb = g.Tb;
    P.Tw = g.Tw;
    P.Wt = g.Wt;
    P.nty = (P.H + g.Tb - 1) / g.Tb;
    P.ntx = (P.W + g.Tw - 1) / g.Tw;
    P.rowsA = g.rowsA;
    P.rowsB = g.rowsB;
    P.tmem_cols = g.tmem_cols;
    P.in = in;
    if (res) P.res = *res;
    for (int j = 0; j < L; j++) {
        const Layer &ly = p->layers[sg.first + j];
        TcLayer &T = P.layer[j];
        T.w = (const __nv_bfloat16 *)(ws + ly.tc_w_off);
        T.bias = (const float *)(ws + ly.b_off);
        T.relu = ly.L.relu;
        T.res = sg.res_tensor[j] >= 0;
        if (j == L - 1) {
            T.out = out;
        } else {
            bdl_layout lo;
            bdl_layout_init(&lo, 2, ly.out_ext[0], ly.L.cout, 1, ly.out_ext[2], ly.out_ext[3], p->in_layout.Bn, 1,
                            p->in_layout.Bh, p->in_layout.Bw, BDL_BF16);
            T.out = make_view(lo, ws + sg.memo_off[j]);
        }
        P.task_base[j] = sg.task_base[j];
    }
    P.status = (int *)(ws + sg.status_off);
    P.counters = (unsigned long long *)(ws + sg.counter_off);
    P.ntiles = (long long)P.N * P.nty * P.ntx;
    {
        const char *e = getenv("BDL_TRACE");
        if (e && atoi(e) > 0) {
            P.trace_cap = atoi(e);
            if (!trace_buf) cudaMalloc(&trace_buf, (size_t)P.trace_cap * 7 * 8);
            P.trace = trace_buf;
        }
    }
    switch (P.C) {
        case 16: return launch_tc_C<16>(p, sg, P, g, mode, s, launches);
        case 32: return launch_tc_C<32>(p, sg, P, g, mode, s, launches);
        case 64: return launch_tc_C<64>(p, sg, P, g, mode, s, launches);
        case 128: return launch_tc_C<128>(p, sg, P, g, mode, s, launches);
    }
    return fail(BDL_EUNSUPPORTED, "tcgen05 band kernel: channel count");
}

}  // namespace bdl

// Debug: copy the task trace (7 x u64 per task) to host; returns records copied.
extern "C" int bdl_debug_trace_copy(unsigned long long *host, int max_records) {
    if (!bdl::trace_buf || max_records <= 0) return 0;
    cudaDeviceSynchronize();
    cudaMemcpy(host, bdl::trace_buf, (size_t)max_records * 7 * 8, cudaMemcpyDeviceToHost);
    return max_records;
}
