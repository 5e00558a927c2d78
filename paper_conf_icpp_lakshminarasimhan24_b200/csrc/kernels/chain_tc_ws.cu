// Warp-specialized persistent tcgen05 kernel for MEMOIZED (and unmerged) merged execution of 3x3
// conv chains (§3.2.2, Fig 2d, Fig 5), bf16 in / fp32 accumulate.
//
// One CTA per SM, three roles connected by mbarrier pipelines:
//   warps 0-1  scheduler + loader: lane 0 of warp 0 draws tasks (layer, tile) from a ticket counter
//              that walks a host-built, locality-aware wavefront order (layer l of tile row b is
//              scheduled `lag` tile rows after layer l-1 -- the paper's future-work "locality-aware
//              memoization", L1785-1791), claims each task with the three-state CAS protocol
//              (0 -> 1, L513-531), claims not-started dependencies first (recursion, Fig 2d) and
//              waits for in-progress ones (state 1 -> spin until 2).  Both warps then stage the
//              task's input tile (Tb+2 rows x Tw+2 cols x C) into one of two shared-memory buffers.
//   warp 2     MMA issuer: 9 taps x C/16 k-steps x ntiles tcgen05.mma (M=128 pixels, N=C, K=16) per
//              task into one of two TMEM accumulators; weights stream through a 3-stage TMA ring.
//   warps 3-6  epilogue: tcgen05.ld -> +bias (+residual) -> ReLU -> bf16, coalesced bricked stores
//              through a swizzled staging buffer, then release-publish the task (state 2).
// Loads of task i+1, MMAs of task i and the epilogue of task i-1 overlap.
#include <algorithm>
#include <cstdlib>
#include <random>
#include <cstring>
#include <string>
#include <vector>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "common.cuh"
#include "tc_ptx.cuh"

namespace bdl {

namespace ws {

constexpr int kSchedWarp = 0;
constexpr int kLoadWarp0 = 1;
constexpr int kEpiWarps = 16;     // TMEM lane quadrant = warp % 4, four warps per quadrant (one M tile each)

// Warp roles.  C % 64 == 0: the input tile is staged by TMA (one loader warp issues the copies) into
// 128-B-swizzled pixel rows; otherwise four loader warps copy 16-B chunks with cp.async into
// unswizzled chunk planes.
template <int C>
struct Roles {
    static constexpr bool TMA = C % 64 == 0;
    static constexpr int LW = TMA ? 1 : 4;                 // loader warps
    static constexpr int WPROD = kLoadWarp0 + LW;          // weight producer warp (TMA bulk copies)
    static constexpr int MMA = WPROD + 1;                  // MMA warp
    static constexpr int STORE = MMA + 1;                  // output store + memo publication warp
    static constexpr int EPI0 = STORE + 1;                 // first epilogue warp
    static constexpr int THREADS = 32 * (EPI0 + kEpiWarps);
    static constexpr int LOADT = 32 * LW;
};
constexpr int kTPS = 2;           // 3x3 taps per weight stage
constexpr int kSPT = (9 + kTPS - 1) / kTPS;  // weight stages per task
constexpr int kWS = 3;            // weight ring stages
constexpr int kQ = 4;             // scheduler -> loader queue
constexpr int kRing = 8;          // task descriptor ring (loader -> MMA -> epilogue)
constexpr int kStack = 160;
constexpr int kMaxIn = 4;        // input tile buffers (loader runs up to kMaxIn-1 tasks ahead of the MMAs)

struct Layer {
    const __nv_bfloat16 *w;  // packed [9][C/8][C][8]
    const float *bias;
    int relu, res;
    TView out;
};

struct Params {
    CUtensorMap tm_row[kMaxLayers];   // 5-D TMA map of each layer's source (identity BrickMap): box = one
                                      // tile row = Tw/Bw brick-row segments of consecutive bricks
    CUtensorMap tm_seg[kMaxLayers];   // 2-D [pixels][C] map, box = one brick-row segment (any BrickMap)
    CUtensorMap tm_out[kMaxLayers];   // 5-D row maps of each layer's output (TMA epilogue stores)
    CUtensorMap tm_res;               // 5-D row map of the residual tensor
    int row_tma;                      // 1: tm_row usable (bricks of a row are consecutive in memory)
    __nv_bfloat16 *dense;             // non-null: the LAST layer writes dense NCHW [N][C][H][W] here instead of bricks
                                      // (unbrickify fused into the epilogue, bdl_run_dense)
    int L, C;
    int H, W;
    int Tb, Tw, Wt;
    int nty, ntx;
    int lBh, lBw;            // log2 brick extents
    int rowsA;
    int stage_off;           // TMA path: byte offset of the epilogue staging tile (Tb x Wt rows x C*2 B)
    int nin, nacc;           // input buffers (1-2), accumulators (1-2)
    int ntl;                 // M tiles per task
    int tmem_cols;
    Layer layer[kMaxLayers];
    TView in, res;
    int *status;
    long long task_base[kMaxLayers];
    unsigned long long *counters;   // run state (common.cuh run_epoch / run_exit); [7] debug trace index
    const int *order;               // encoded (l << 24) | tile, or null (unmerged: identity over only_layer)
    long long norder;
    int only_layer;
    unsigned long long *trace;      // debug: 8 x u64 per task, or null
    int trace_cap;
    int dbg;                        // debug timing knobs (BDL_WS_DBG): 1 = no MMA, 2 = no epilogue math/stores,
                                    // 8 = weights not re-streamed, 16 = residual not fetched (all give wrong results)
};

struct Shared {
    uint64_t q_full[kQ], q_empty[kQ];
    uint64_t res_full, stg_free;
    uint64_t in_full[kMaxIn], in_empty[kMaxIn], acc_full[2], acc_empty[2], wfull[kWS], wempty[kWS];
    uint32_t tmem_base;
    int q_l[kQ];
    long long q_t[kQ];
    int desc_l[kRing];
    long long desc_t[kRing];
    uint64_t desc_full[kRing];   // completes (phase seq / kRing) once desc_*[slot] holds task seq
    unsigned long long tr[kRing][8];   // debug trace timestamps per task slot
    int stk_l[kStack];
    long long stk_t[kStack];
};

__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ int *status_word(const Params &p, int l, long long t) { return p.status + p.task_base[l] + t; }

__device__ __forceinline__ void decode(const Params &p, long long t, int &n, int &ty, int &tx) {
    tx = (int)(t % p.ntx);
    t /= p.ntx;
    ty = (int)(t % p.nty);
    n = (int)(t / p.nty);
}

// Element offset of channel 0 of pixel (n, y, x) in a bricked 2-D view with power-of-two bricks.
__device__ __forceinline__ long long pix_off(const TView &v, int lBh, int lBw, int n, int y, int x) {
    int by = y >> lBh, bx = x >> lBw;
    long long logical = ((long long)n * v.nb[2] + by) * v.nb[3] + bx;
    long long phys = v.bmap ? (long long)v.bmap[logical] : logical;
    return phys * v.brick_elems + (long long)(((y - (by << lBh)) << lBw) + (x - (bx << lBw))) * v.Cp;
}

// dependency k (0..8) of tile t: layer l-1 tile (n, ty+dy, tx+dx)
__device__ __forceinline__ bool dep_of(const Params &p, long long t, int k, long long &dt) {
    int n, ty, tx;
    decode(p, t, n, ty, tx);
    int qy = ty + k / 3 - 1, qx = tx + k % 3 - 1;
    if (k >= 9 || qy < 0 || qy >= p.nty || qx < 0 || qx >= p.ntx) return false;
    dt = ((long long)n * p.nty + qy) * p.ntx + qx;
    return true;
}

__device__ __forceinline__ int tag_state(int v, unsigned EP) { return ((v & ~3) == (int)EP) ? (v & 3) : 0; }

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ptx::smem_u32(bar)) : "memory");
}

// ---------------------------------------------------------------------------------------------- loader
// Stage the (Tb+2) x (Tw+2) pixel input tile of a task into C/8 chunk planes.  Work is split into
// brick-row segments (Bw contiguous pixels = Bw*C*2 contiguous bytes in the bricked tensor) plus the
// two halo pixels of each row; address arithmetic (incl. the BrickMap lookup) is done once per
// segment, and the lanes of a warp copy the segment's 16-byte chunks with cp.async (zero-filled
// outside the image).
template <int C>
__device__ __forceinline__ void load_tile(const Params &p, const TView &src_in, int n, int y0, int x0, uint8_t *buf,
                                          int tidl) {
    constexpr int KC = C / 8;
    constexpr int LKC = KC == 2 ? 1 : KC == 4 ? 2 : KC == 8 ? 3 : 4;
    const int lane = tidl & 31, wl = tidl >> 5;
    // hoist the view into registers
    const __nv_bfloat16 *base = reinterpret_cast<const __nv_bfloat16 *>(src_in.ptr);
    const int32_t *bmap = src_in.bmap;
    const long long be = src_in.brick_elems;
    const int nb2 = src_in.nb[2], nb3 = src_in.nb[3], Cp = src_in.Cp;
    const int Bw = 1 << p.lBw, Bh = 1 << p.lBh;
    const int R = p.Tb + 2, Wt = p.Wt;
    const int nseg = p.Tw >> p.lBw;            // full brick segments per row
    const int items = R * (nseg + 2);          // + left / right halo pixel
    const uint32_t rowsA16 = (uint32_t)p.rowsA * 16;
    for (int it = wl; it < items; it += Roles<C>::LW) {
        const int a = it / (nseg + 2), sg = it - a * (nseg + 2);
        const int y = y0 - 1 + a;
        int xs, npx, q0;                           // first image column, pixels, first tile column
        if (sg == 0) { xs = x0 - 1; npx = 1; q0 = 0; }
        else if (sg == nseg + 1) { xs = x0 + p.Tw; npx = 1; q0 = Wt - 1; }
        else { xs = x0 + (sg - 1) * Bw; npx = Bw; q0 = 1 + (sg - 1) * Bw; }
        const bool rok = y >= 0 && y < p.H;
        long long seg_off = 0;
        if (rok && xs >= 0 && xs < p.W) {
            const int by = y >> p.lBh, bx = xs >> p.lBw;
            long long logical = ((long long)n * nb2 + by) * nb3 + bx;
            long long phys = bmap ? (long long)bmap[logical] : logical;
            seg_off = phys * be + (long long)(((y - by * Bh) << p.lBw) + (xs - bx * Bw)) * Cp;
        }
        const int nchunk = npx * KC;
        for (int c = lane; c < nchunk; c += 32) {
            const int px = c >> LKC, k = c & (KC - 1);
            const int x = xs + px;
            const bool ok = rok && x >= 0 && x < p.W;
            const void *g = ok ? (const void *)(base + seg_off + (long long)px * Cp + k * 8) : (const void *)base;
            ptx::cp_async16(buf + k * rowsA16 + (uint32_t)(a * Wt + q0 + px) * 16, g, ok ? 16u : 0u);
        }
    }
    ptx::cp_async_wait_all();
    ptx::fence_proxy_async_smem();
}

// ---------------------------------------------------------------------------------------------- scheduler
// Warp-cooperative: draws tickets along the wavefront order, claims tasks (CAS 0 -> 1), claims their
// not-started dependencies recursively (Fig 2d) -- the 9 dependency tags of a task are read and
// CAS-ed by 9 lanes at once -- and hands claimed tasks to the loaders, dependencies first.
__device__ void scheduler(const Params &p, Shared &sh) {
    const int lane = threadIdx.x % 32;
    const unsigned EP = run_epoch(p.counters) << 2;
    const bool unmerged = p.only_layer >= 0;
    unsigned long long oks = 0, fails = 0;
    int sp = 0;
    uint32_t qseq = 0;
    auto emit = [&](int l, long long t) {
        const int slot = qseq % kQ;
        if (qseq >= (uint32_t)kQ) ptx::mbar_wait(&sh.q_empty[slot], ((qseq / kQ) - 1) & 1);
        if (lane == 0) {
            sh.q_l[slot] = l;
            sh.q_t[slot] = t;
            mbar_arrive(&sh.q_full[slot]);
        }
        __syncwarp();
        qseq++;
    };
    for (;;) {
        if (sp == 0) {
            unsigned long long tk = 0;
            if (lane == 0) tk = atomicAdd(&p.counters[4], 1ULL);
            tk = __shfl_sync(0xffffffff, tk, 0);
            if ((long long)tk >= p.norder) break;
            int l;
            long long t;
            if (unmerged) {
                l = p.only_layer;
                t = (long long)tk;
            } else {
                int e = p.order[tk];
                l = e >> 24;
                t = e & 0xFFFFFF;
                int ok = 0;
                if (lane == 0) {
                    int *sw = status_word(p, l, t);
                    int cur = ld_acquire(sw);
                    ok = tag_state(cur, EP) == 0 && atomicCAS(sw, cur, (int)(EP | 1)) == cur;
                }
                ok = __shfl_sync(0xffffffff, ok, 0);
                if (!ok) continue;  // already claimed by a dependent
                oks++;
            }
            if (lane == 0) {
                sh.stk_l[0] = l;
                sh.stk_t[0] = t;
            }
            sp = 1;
            if (!unmerged) {
                for (int s = 0; s < sp; s++) {
                    __syncwarp();
                    const int sl = sh.stk_l[s];
                    const long long st = sh.stk_t[s];
                    if (sl == 0) continue;
                    long long dt = 0;
                    int claimed = 0, busy = 0;
                    if (dep_of(p, st, lane, dt)) {
                        int *dw = status_word(p, sl - 1, dt);
                        int cur = ld_acquire(dw);
                        int s2 = tag_state(cur, EP);
                        if (s2 == 0 && atomicCAS(dw, cur, (int)(EP | 1)) == cur) claimed = 1;
                        else if (s2 != 2) busy = 1;
                    }
                    unsigned cm = __ballot_sync(0xffffffff, claimed);
                    fails += __popc(__ballot_sync(0xffffffff, busy));
                    oks += __popc(cm);
                    if (claimed) {
                        int pos = sp + __popc(cm & ((1u << lane) - 1));
                        if (pos < kStack) {
                            sh.stk_l[pos] = sl - 1;
                            sh.stk_t[pos] = dt;
                        }
                    }
                    sp += __popc(cm);
                }
                __syncwarp();
            }
        }
        sp--;
        __syncwarp();
        emit(sh.stk_l[sp], sh.stk_t[sp]);
    }
    emit(-1, 0);
    if (lane == 0) {
        if (oks) atomicAdd(&p.counters[1], oks);
        if (fails) atomicAdd(&p.counters[2], fails);
    }
}

// ---------------------------------------------------------------------------------------------- mma
// Weights stream through a kWS-stage ring, kTPS taps (kTPS x C x C bf16) per stage; global stage index
// g = kSPT*seq + j -> ring slot g % kWS; filled by the weight-producer warp, released by tcgen05.commit.
// The MMA warp runs converged so that descriptors are warp-uniform (uniform registers); an elected lane
// issues each MMA.
template <int C>
__device__ __forceinline__ void issue_task(const Params &p, Shared &sh, uint32_t a_base, uint32_t d_base, uint8_t *wst,
                                           uint32_t seq) {
    constexpr uint32_t WB = C * C * 2;   // one tap
    constexpr uint32_t LBO_B = C * 16;
    constexpr uint32_t IDESC = ptx::idesc_bf16_f32(128, C);
    const uint32_t LBO_A = (uint32_t)p.rowsA * 16;
    const uint32_t w_base = ptx::smem_u32(wst);
    constexpr bool SW = Roles<C>::TMA;
    // TMA layout: [C/64 k-blocks][rows][128 B] 128-B swizzled, SBO = 8 rows x 128 B;
    // cp.async layout: [C/8 chunk planes][rows][16 B] unswizzled, LBO = plane stride, SBO = 128 B.
    const uint64_t adesc0 = SW ? ptx::umma_desc_sw128(0, 1024) : ptx::umma_desc_noswz(0, LBO_A, 128);
    const uint64_t bdesc0 = ptx::umma_desc_noswz(0, LBO_B, 128);
    const uint32_t row_u = SW ? 8 : 1;                                     // 16-B units per pixel row
    const uint32_t kb_u = SW ? (uint32_t)p.rowsA * 8 : 0;                  // 16-B units per k-block
    for (int j = 0; j < kSPT; j++) {
        const uint32_t g = kSPT * seq + j;
        const int st = g % kWS;
        ptx::mbar_wait(&sh.wfull[st], (g / kWS) & 1);
        ptx::tc_fence_after();
        for (int tq = 0; tq < kTPS && j * kTPS + tq < 9; tq++) {
            const int tap = j * kTPS + tq;
            const uint32_t shift = (uint32_t)((tap / 3) * p.Wt + (tap % 3));
            const uint32_t b0 = (w_base + st * (kTPS * WB) + tq * WB) >> 4;
            const uint32_t a0 = (a_base >> 4) + shift * row_u;
            for (int t = 0; t < p.ntl; t++) {
#pragma unroll
                for (int kk = 0; kk < C / 16; kk++) {
                    const uint32_t koff = SW ? (kk / 4) * kb_u + (kk % 4) * 2 : kk * (LBO_A >> 3);
                    const uint64_t ad = adesc0 | (uint64_t)((a0 + t * 128 * row_u + koff) & 0x3FFF);
                    const uint64_t bd = bdesc0 | (uint64_t)((b0 + kk * (LBO_B >> 3)) & 0x3FFF);
                    ptx::mma_bf16_elect(d_base + t * C, ad, bd, IDESC, (tap | kk) != 0);
                }
            }
        }
        ptx::mma_commit_elect(&sh.wempty[st]);
    }
}

__device__ __forceinline__ uint32_t pack2(float a, float b) {
    __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<uint32_t *>(&v);
}

// ---------------------------------------------------------------------------------------------- kernel
// TMA path.  Each in-image tile row is fetched by ONE 5-D TMA box (Tw/Bw consecutive bricks x one
// brick row x 64 channels, 128-B swizzled) when the BrickMap is the identity, else one 2-D TMA per
// brick-row segment; the two halo pixels of a row are copied with cp.async into the same swizzled
// layout; rows and halo pixels outside the image are zero-filled.  The UMMA descriptor applies the
// same absolute-address swizzle, so a tap shift of any number of pixel rows is a start-address offset.
template <int C>
__device__ __forceinline__ void load_tile_tma(const Params &p, int src_l, const TView &src, int n, int y0, int x0,
                                              uint8_t *buf, uint64_t *bar, int lane) {
    constexpr int KB = C / 64;
    const int32_t *bmap = src.bmap;
    const int nb2 = src.nb[2], nb3 = src.nb[3];
    const int Bw = 1 << p.lBw, Bh = 1 << p.lBh;
    const int R = p.Tb + 2, Wt = p.Wt;
    const int nseg = p.Tw >> p.lBw;
    const uint32_t kb_stride = (uint32_t)p.rowsA * 128;
    const __nv_bfloat16 *base = reinterpret_cast<const __nv_bfloat16 *>(src.ptr);
    const int per_row = p.row_tma ? 1 : nseg;
    // (a) bulk rows / segments by TMA, zero rows outside the image
    for (int it = lane; it < R * per_row; it += 32) {
        const int a = it / per_row, sg = it - a * per_row;
        const int y = y0 - 1 + a;
        uint8_t *dst = buf + (size_t)(a * Wt + 1 + sg * Bw) * 128;
        if (y >= 0 && y < p.H) {
            const int by = y >> p.lBh, yin = y - by * Bh;
            const int bx0 = (x0 >> p.lBw) + sg;
            if (p.row_tma) {
                const uint32_t bytes = (uint32_t)p.Tw * 128;
#pragma unroll
                for (int kb = 0; kb < KB; kb++) {
                    ptx::mbar_expect_tx(bar, bytes);
                    ptx::tma_load_5d(dst + kb * kb_stride, &p.tm_row[src_l], kb * 64, 0, bx0, yin, n * nb2 + by, bar);
                }
            } else if ((bx0 << p.lBw) < p.W) {
                const long long logical = ((long long)n * nb2 + by) * nb3 + bx0;
                const long long phys = bmap ? (long long)bmap[logical] : logical;
                const int pix = (int)(phys * (Bh * Bw) + (yin << p.lBw));
#pragma unroll
                for (int kb = 0; kb < KB; kb++) {
                    ptx::mbar_expect_tx(bar, (uint32_t)Bw * 128);
                    ptx::tma_load_2d(dst + kb * kb_stride, &p.tm_seg[src_l], kb * 64, pix, bar);
                }
            } else {
                for (int kb = 0; kb < KB; kb++)
                    for (int q = 0; q < Bw * 8; q++)
                        *reinterpret_cast<uint4 *>(dst + kb * kb_stride + q * 16) = make_uint4(0, 0, 0, 0);
            }
        } else {
            const int npx = p.row_tma ? p.Tw : Bw;
            for (int kb = 0; kb < KB; kb++)
                for (int q = 0; q < npx * 8; q++)
                    *reinterpret_cast<uint4 *>(dst + kb * kb_stride + q * 16) = make_uint4(0, 0, 0, 0);
        }
    }
    // (b) halo pixels (columns x0-1 and x0+Tw): 16-B chunks with cp.async, swizzled by address
    constexpr int CH = C / 8;
    for (int it = lane; it < R * 2 * CH; it += 32) {
        const int k = it % CH, hp = it / CH;
        const int a = hp >> 1, side = hp & 1;
        const int y = y0 - 1 + a, x = side ? x0 + p.Tw : x0 - 1;
        const int q = a * Wt + (side ? Wt - 1 : 0);
        uint8_t *row = buf + (k / 8) * kb_stride + (size_t)q * 128;
        const uint32_t sw = (((ptx::smem_u32(row) >> 7) & 7) ^ (k & 7)) * 16;
        const bool ok = y >= 0 && y < p.H && x >= 0 && x < p.W;
        const void *g = base;
        if (ok) g = base + pix_off(src, p.lBh, p.lBw, n, y, x) + k * 8;
        ptx::cp_async16(row + sw, g, ok ? 16u : 0u);
    }
    ptx::cp_async_wait_all();
    ptx::fence_proxy_async_smem();
    __syncwarp();
}

template <int C>
__global__ void __launch_bounds__(Roles<C>::THREADS, 1) memo_ws_kernel(const __grid_constant__ Params p) {
    using RL = Roles<C>;
    constexpr int kThreads = RL::THREADS, kMmaWarp = RL::MMA, kEpiWarp0 = RL::EPI0, kLoadThreads = RL::LOADT;
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ Shared sh;
    constexpr int KC = C / 8;
    // warp index via shuffle: provably warp-uniform, so role branches keep the uniform datapath
    const int warp = __shfl_sync(0xffffffff, (int)threadIdx.x / 32, 0), lane = threadIdx.x % 32;
    const size_t in_bytes = (size_t)KC * p.rowsA * 16;
    const size_t stage_bytes = RL::TMA ? (((size_t)(C / 64) * p.Tb * p.Wt * 128 + 1023) / 1024 * 1024) : 0;
    uint8_t *wst = smem + in_bytes * p.nin + stage_bytes;
    float *bias_s = reinterpret_cast<float *>(wst + kWS * kTPS * C * C * 2);  // [L][C]
    for (int i = threadIdx.x; i < p.L * C; i += kThreads) bias_s[i] = p.layer[i / C].bias[i % C];
    if (RL::TMA && (ptx::smem_u32(smem) & 1023)) __trap();  // 128-B swizzle atoms need 1024-B alignment

    if (threadIdx.x == 0) {
        for (int i = 0; i < kQ; i++) {
            ptx::mbar_init(&sh.q_full[i], 1);
            ptx::mbar_init(&sh.q_empty[i], 2);   // loader + weight producer
        }
        for (int i = 0; i < kMaxIn; i++) {
            ptx::mbar_init(&sh.in_full[i], 1);
            ptx::mbar_init(&sh.in_empty[i], 1);
        }
        for (int i = 0; i < 2; i++) {
            ptx::mbar_init(&sh.acc_full[i], 1);
            ptx::mbar_init(&sh.acc_empty[i], kEpiWarps);   // one arrival per epilogue warp
        }
        for (int i = 0; i < kWS; i++) {
            ptx::mbar_init(&sh.wfull[i], 1);
            ptx::mbar_init(&sh.wempty[i], 1);
        }
        ptx::mbar_init(&sh.res_full, 1);
        ptx::mbar_init(&sh.stg_free, 1);
        for (int i = 0; i < kRing; i++) ptx::mbar_init(&sh.desc_full[i], 1);
        ptx::fence_barrier_init();
    }
    if (warp == kMmaWarp) {
        ptx::tmem_alloc(&sh.tmem_base, p.tmem_cols);
        ptx::tmem_relinquish();
    }
    // (guard rows of the input buffers are never written by the loader; they only feed accumulator rows
    //  that the epilogue discards, and MMA rows are independent, so they need no initialization)
    ptx::fence_proxy_async_smem();
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    pdl_launch_dependents();  // let the next kernel (unbrickify) get scheduled
    // PDL: only the roles that touch the previous kernel's output (the subgraph input) or the memo tags wait for
    // it; the weight producer (packed weights) starts right away.
    // (the scheduler too: it rewrites memo tags that a previous run of this subgraph may still be waiting on)
    const bool reads_input = (warp >= kLoadWarp0 && warp < RL::WPROD) || warp == RL::STORE ||
                             (!RL::TMA && warp >= kEpiWarp0) || warp == kSchedWarp;
    if (reads_input) pdl_wait();

    if (warp == kSchedWarp) {
        scheduler(p, sh);
    } else if (warp < RL::WPROD) {
        // ------------------------------------------------------------------ loaders
        const int tidl = threadIdx.x - 32 * kLoadWarp0;
        const unsigned EP = run_epoch(p.counters) << 2;
        for (uint32_t seq = 0;; seq++) {
            const int slot = seq % kQ;
            ptx::mbar_wait(&sh.q_full[slot], (seq / kQ) & 1);
            const int l = sh.q_l[slot];
            const long long t = sh.q_t[slot];
            const unsigned long long t_q = gtime();
            const int b = seq % p.nin;
            if (seq >= (uint32_t)p.nin) ptx::mbar_wait(&sh.in_empty[b], ((seq / p.nin) - 1) & 1);
            unsigned long long t_dep = 0;
            if (l >= 0) {
                if (warp == kLoadWarp0 && l > 0 && p.only_layer < 0) {
                    // wait for the 9 dependency tags in parallel (state 2 of this epoch)
                    long long dt;
                    unsigned long long spins = 0;
                    if (dep_of(p, t, lane, dt)) {
                        const int *dw = status_word(p, l - 1, dt);
                        while (ld_acquire(dw) != (int)(EP | 2)) {
                            spins++;
                            __nanosleep(32);
                        }
                    }
                    __syncwarp();
                    for (int o = 16; o; o >>= 1) spins += __shfl_xor_sync(0xffffffff, spins, o);
                    if (lane == 0 && spins) atomicAdd(&p.counters[3], spins);
                }
                asm volatile("bar.sync 1, %0;" ::"n"(kLoadThreads) : "memory");
                if constexpr (RL::TMA) ptx::fence_proxy_async();  // acquired data is read by TMA (async proxy)
                t_dep = gtime();
                int n, ty, tx;
                decode(p, t, n, ty, tx);
                const TView &src = l == 0 ? p.in : p.layer[l - 1].out;
                if constexpr (RL::TMA)
                    load_tile_tma<C>(p, l, src, n, ty * p.Tb, tx * p.Tw, smem + in_bytes * b, &sh.in_full[b], lane);
                else
                    load_tile<C>(p, src, n, ty * p.Tb, tx * p.Tw, smem + in_bytes * b, tidl);
            }
            asm volatile("bar.sync 1, %0;" ::"n"(kLoadThreads) : "memory");
            if (warp == kLoadWarp0 && lane == 0) {
                sh.desc_l[seq % kRing] = l;
                sh.desc_t[seq % kRing] = t;
                sh.tr[seq % kRing][0] = t_q;
                sh.tr[seq % kRing][1] = t_dep;
                sh.tr[seq % kRing][2] = gtime();
                mbar_arrive(&sh.desc_full[seq % kRing]);   // release: descriptor visible to its waiters
                mbar_arrive(&sh.in_full[b]);
                mbar_arrive(&sh.q_empty[slot]);
            }
            if (l < 0) break;
        }
    } else if (warp == RL::WPROD) {
        // ------------------------------------------------------------------ weight producer
        // follows the scheduler queue (task layers are known before the inputs land) and keeps the
        // kWS-stage ring full, one 3x3 tap (C x C bf16) per stage
        for (uint32_t seq = 0;; seq++) {
            const int slot = seq % kQ;
            ptx::mbar_wait(&sh.q_full[slot], (seq / kQ) & 1);
            const int l = sh.q_l[slot];
            __syncwarp();
            if (lane == 0) mbar_arrive(&sh.q_empty[slot]);
            if (l < 0) break;
            const __nv_bfloat16 *w = p.layer[l].w;
            for (int j = 0; j < kSPT; j++) {
                const uint32_t g = kSPT * seq + j;
                const int st = g % kWS;
                const int ntap = min(kTPS, 9 - j * kTPS);
                const uint32_t bytes = (uint32_t)ntap * C * C * 2;
                if (g >= (uint32_t)kWS) ptx::mbar_wait(&sh.wempty[st], ((g / kWS) - 1) & 1);
                if (ptx::elect_one()) {
                    if ((p.dbg & 8) && seq >= 4) {
                        mbar_arrive(&sh.wfull[st]);   // debug: weights not re-streamed (wrong results)
                    } else {
                        ptx::mbar_arrive_expect_tx(&sh.wfull[st], bytes);
                        ptx::bulk_g2s(wst + st * (kTPS * C * C * 2), w + (size_t)j * kTPS * C * C, bytes, &sh.wfull[st]);
                    }
                }
                __syncwarp();
            }
        }
    } else if (warp == kMmaWarp) {
        // ------------------------------------------------------------------ MMA issuer
        const uint32_t acc_cols = (uint32_t)p.ntl * C;
        const uint32_t tmem_base = __shfl_sync(0xffffffff, sh.tmem_base, 0);
        for (uint32_t seq = 0;; seq++) {
            const int b = seq % p.nin, a = seq % p.nacc;
            ptx::mbar_wait(&sh.in_full[b], (seq / p.nin) & 1);
            const int l = sh.desc_l[seq % kRing];
            if (seq >= (uint32_t)p.nacc) ptx::mbar_wait(&sh.acc_empty[a], ((seq / p.nacc) - 1) & 1);
            if (l < 0) {
                if (lane == 0) mbar_arrive(&sh.acc_full[a]);
                break;
            }
            ptx::tc_fence_after();
            if (lane == 0) sh.tr[seq % kRing][3] = gtime();
            if (!(p.dbg & 1)) issue_task<C>(p, sh, ptx::smem_u32(smem + in_bytes * b), tmem_base + a * acc_cols, wst, seq);
            if (lane == 0) sh.tr[seq % kRing][4] = gtime();
            ptx::mma_commit_elect(&sh.in_empty[b]);
            ptx::mma_commit_elect(&sh.acc_full[a]);
            __syncwarp();
        }
    } else {
        // ------------------------------------------------------------------ epilogue + store warps
        // Epilogue: kEpiWarps warps; warp ew reads TMEM lane quadrant warp % 4 of M tiles ew/4, ew/4+4,..
        // Each thread owns one pixel (TMEM lane) and processes its channels 32 at a time.
        // TMA path: a dedicated staging tile (128-B swizzled pixel rows m = i*Wt + j) receives the
        // residual rows by TMA as soon as the task is known (overlapping its MMAs), each thread reads its
        // pixel's residual and writes its result there, and the store warp TMA-stores whole tile rows
        // into the bricked output, frees the staging tile, and publishes the task (memo state 2) once
        // its global writes are complete.
        const int Hg = p.layer[0].out.nb[2] << p.lBh;  // all layers share the spatial grid
        constexpr int CB = C < 32 ? C : 32;            // channels per TMEM load batch
        uint8_t *stg = smem + p.stage_off;
        const uint32_t stg_kb = (uint32_t)p.Tb * p.Wt * 128;   // staging bytes per 64-channel block
        if (warp == RL::STORE) {
            // Per task i: wait for its descriptor; once the previous task's TMA store has read the
            // staging tile, free it and immediately prefetch task i's residual rows into it; then
            // publish the previous task after its global writes complete; then wait for the epilogue
            // and issue task i's row stores.
            int prev_l = -1;
            long long prev_t = 0;
            uint32_t prev_seq = 0;
            unsigned long long prev_sync = 0, prev_read = 0;
            const unsigned EPs = run_epoch(p.counters) << 2;
            auto publish = [&](int l, long long t, uint32_t sq, unsigned long long t_sync, unsigned long long t_read) {
                if (p.only_layer < 0) {
                    __threadfence();
                    st_release(status_word(p, l, t), (int)(EPs | 2));
                }
                atomicAdd(&p.counters[0], 1ULL);
                if (p.trace) {
                    unsigned long long k = atomicAdd(&p.counters[7], 1ULL);
                    if (k < (unsigned long long)p.trace_cap) {
                        unsigned smid;
                        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
                        unsigned long long *rec = p.trace + k * 16;
                        rec[0] = ((unsigned long long)smid << 40) | ((unsigned long long)blockIdx.x << 8) | (unsigned)l;
                        rec[1] = (unsigned long long)t;
                        for (int f = 0; f < 7; f++) rec[2 + f] = sh.tr[sq % kRing][f];
                        rec[9] = t_sync;
                        rec[10] = t_read;
                        rec[11] = gtime();
                    }
                }
            };
            for (uint32_t seq = 0;; seq++) {
                if (lane == 0 && RL::TMA && prev_l >= 0) {
                    ptx::bulk_wait_read0();              // previous task's staging read out
                    prev_read = gtime();
                    mbar_arrive(&sh.stg_free);
                }
                // wait for this task's descriptor; if it is not there yet, publish the previous task first
                // (the loader may be waiting for exactly that publication: never hold it back)
                while (!ptx::mbar_test(&sh.desc_full[seq % kRing], (seq / kRing) & 1)) {
                    if (lane == 0 && prev_l >= 0) {
                        if constexpr (RL::TMA) {
                            ptx::bulk_wait0();
                            ptx::fence_proxy_async();
                        }
                        publish(prev_l, prev_t, prev_seq, prev_sync, prev_read);
                        prev_l = -1;
                    }
                    __nanosleep(20);
                }
                prev_l = __shfl_sync(0xffffffff, prev_l, 0);
                const int l = sh.desc_l[seq % kRing];
                const long long t = sh.desc_t[seq % kRing];
                if (lane == 0) {
                    if (RL::TMA && l >= 0 && p.layer[l].res && !(p.dbg & 16)) {  // prefetch this task's residual rows
                        const Layer &ly = p.layer[l];
                        int n, ty, tx;
                        decode(p, t, n, ty, tx);
                        const int y0 = ty * p.Tb, x0 = tx * p.Tw;
                        const int nrows = min(p.Tb, p.H - y0);
                        for (int i = 0; i < nrows; i++) {
                            const int y = y0 + i;
                            for (int kb = 0; kb < C / 64; kb++) {
                                ptx::mbar_expect_tx(&sh.res_full, (uint32_t)p.Tw * 128);
                                ptx::tma_load_5d(stg + kb * stg_kb + (size_t)i * p.Wt * 128, &p.tm_res, kb * 64, 0,
                                                 x0 >> p.lBw, y & ((1 << p.lBh) - 1), n * ly.out.nb[2] + (y >> p.lBh),
                                                 &sh.res_full);
                            }
                        }
                        mbar_arrive(&sh.res_full);
                    } else if (RL::TMA && l >= 0 && p.layer[l].res) {
                        mbar_arrive(&sh.res_full);   // debug 16: residual not fetched (wrong results)
                    }
                    if (prev_l >= 0) {
                        if constexpr (RL::TMA) {
                            ptx::bulk_wait0();           // global writes performed
                            ptx::fence_proxy_async();
                        }
                        publish(prev_l, prev_t, prev_seq, prev_sync, prev_read);
                    }
                }
                __syncwarp();
                prev_l = -1;
                if (l < 0) break;
                const Layer &ly = p.layer[l];
                int n, ty, tx;
                decode(p, t, n, ty, tx);
                const int y0 = ty * p.Tb, x0 = tx * p.Tw;
                // wait until the epilogue warps have written this task's results
                asm volatile("bar.sync 2, %0;" ::"n"(32 * (kEpiWarps + 1)) : "memory");
                prev_sync = gtime();
                if (lane == 0 && RL::TMA && !(p.dense && l == p.L - 1)) {   // (dense output: the epilogue wrote it)
                    for (int i = 0; i < p.Tb && y0 + i < Hg; i++) {
                        const int y = y0 + i;
                        for (int kb = 0; kb < C / 64; kb++)
                            ptx::tma_store_5d(&p.tm_out[l], stg + kb * stg_kb + (size_t)i * p.Wt * 128, kb * 64, 0,
                                              x0 >> p.lBw, y & ((1 << p.lBh) - 1), n * ly.out.nb[2] + (y >> p.lBh));
                    }
                    ptx::bulk_commit();
                }
                prev_l = l;
                prev_t = t;
                prev_seq = seq;
                __syncwarp();
            }
        } else {
            const int ew = warp - kEpiWarp0;
            const int quad = warp % 4;
            const int tile0 = ew / 4;
            const uint32_t acc_cols = (uint32_t)p.ntl * C;
            uint32_t res_phase = 0;
            for (uint32_t seq = 0;; seq++) {
                const int a = seq % p.nacc;
                ptx::mbar_wait(&sh.desc_full[seq % kRing], (seq / kRing) & 1);
                const int l = sh.desc_l[seq % kRing];
                const long long t = sh.desc_t[seq % kRing];
                if (l < 0) break;
                const Layer &ly = p.layer[l];
                int n, ty, tx;
                decode(p, t, n, ty, tx);
                const int y0 = ty * p.Tb, x0 = tx * p.Tw;
                if (RL::TMA && seq > 0) ptx::mbar_wait(&sh.stg_free, (seq - 1) & 1);  // last store read out
                ptx::mbar_wait(&sh.acc_full[a], (seq / p.nacc) & 1);
                if (ew == 0 && lane == 0) sh.tr[seq % kRing][5] = gtime();
                ptx::tc_fence_after();
                if (RL::TMA && ly.res) {
                    ptx::mbar_wait(&sh.res_full, res_phase);
                    res_phase ^= 1;
                }
                __nv_bfloat16 *outp = reinterpret_cast<__nv_bfloat16 *>(ly.out.ptr);
                const __nv_bfloat16 *resp = reinterpret_cast<const __nv_bfloat16 *>(p.res.ptr);
                const bool dn = p.dense != nullptr && l == p.L - 1;
                const int Wg = ly.out.nb[3] << p.lBw;  // bricked grid extents
                const float *bl = bias_s + l * C;
                for (int tile = tile0; tile < ((p.dbg & 2) ? 0 : p.ntl); tile += 4) {
                    const int m = tile * 128 + quad * 32 + lane;
                    const int i = m / p.Wt, j = m - i * p.Wt;
                    const int y = y0 + i, x = x0 + j;
                    // 0: skip (garbage column / outside the tile / outside the grid), 1: zero (masked), 2: value
                    int kind = 0;
                    if (i < p.Tb && j < p.Tw && y < Hg && x < Wg) kind = (y < p.H && x < p.W) ? 2 : 1;
                    const bool has_res = kind == 2 && ly.res;
                    uint8_t *srow = stg + (size_t)m * 128;                       // TMA path staging row
                    const uint32_t sx = (ptx::smem_u32(srow) >> 7) & 7;        // its swizzle phase
                    uint4 *dst = nullptr;
                    uint4 rv[RL::TMA ? 1 : KC];
                    if constexpr (!RL::TMA) {
                        dst = reinterpret_cast<uint4 *>(outp + (kind ? pix_off(ly.out, p.lBh, p.lBw, n, y, x) : 0));
                        if (has_res) {
                            const uint4 *rs = reinterpret_cast<const uint4 *>(resp + pix_off(p.res, p.lBh, p.lBw, n, y, x));
#pragma unroll
                            for (int k = 0; k < KC; k++) rv[k] = __ldcg(rs + k);
                        }
                    }
                    const uint32_t taddr = sh.tmem_base + a * acc_cols + ((uint32_t)(quad * 32) << 16) + tile * C;
#pragma unroll
                    for (int cb = 0; cb < C / CB; cb++) {
                        uint32_t r[CB / 16][16];
#pragma unroll
                        for (int cc = 0; cc < CB / 16; cc++) ptx::tmem_ld16(taddr + cb * CB + cc * 16, r[cc]);
                        ptx::tmem_ld_wait();
#pragma unroll
                        for (int cc = 0; cc < CB / 16; cc++) ptx::reg_fence16(r[cc]);
#pragma unroll
                        for (int kq = 0; kq < CB / 8; kq++) {
                            const int k = cb * (CB / 8) + kq;
                            uint4 *sp = nullptr;
                            if constexpr (RL::TMA) sp = reinterpret_cast<uint4 *>(srow + (k / 8) * stg_kb + (((k & 7) ^ sx) << 4));
                            uint4 o = make_uint4(0, 0, 0, 0);
                            if (kind == 2) {
                                float v[8];
                                const float4 b0 = *reinterpret_cast<const float4 *>(bl + k * 8);
                                const float4 b1 = *reinterpret_cast<const float4 *>(bl + k * 8 + 4);
                                const float bb[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
                                for (int e = 0; e < 8; e++) v[e] = __uint_as_float(r[kq / 2][(kq % 2) * 8 + e]) + bb[e];
                                if (has_res) {
                                    uint4 rr;
                                    if constexpr (RL::TMA) rr = *sp;
                                    else rr = rv[k];
                                    const __nv_bfloat162 *h2 = reinterpret_cast<const __nv_bfloat162 *>(&rr);
#pragma unroll
                                    for (int e = 0; e < 4; e++) {
                                        float2 f = __bfloat1622float2(h2[e]);
                                        v[2 * e] += f.x;
                                        v[2 * e + 1] += f.y;
                                    }
                                }
                                if (ly.relu) {
#pragma unroll
                                    for (int e = 0; e < 8; e++) v[e] = fmaxf(v[e], 0.f);
                                }
                                o = make_uint4(pack2(v[0], v[1]), pack2(v[2], v[3]), pack2(v[4], v[5]), pack2(v[6], v[7]));
                            }
                            if (dn) {
                                // dense NCHW output: lanes hold consecutive pixels of a row, so each channel's store
                                // of the warp is one contiguous segment
                                if (kind == 2) {
                                    const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&o);
                                    __nv_bfloat16 *q = p.dense + (((long long)n * C + k * 8) * p.H + y) * p.W + x;
#pragma unroll
                                    for (int e = 0; e < 8; e++) q[(long long)e * p.H * p.W] = h[e];
                                }
                            } else if constexpr (RL::TMA) {
                                if (kind) *sp = o;
                            } else {
                                if (kind) dst[k] = o;
                            }
                        }
                    }
                }
                ptx::tc_fence_before();
                if (lane == 0) mbar_arrive(&sh.acc_empty[a]);
                if (ew == 0 && lane == 0) sh.tr[seq % kRing][6] = gtime();
                if constexpr (RL::TMA) ptx::fence_proxy_async_smem();
                // hand the task to the store warp (memory ordering of the stores above: bar cumulativity)
                asm volatile("bar.arrive 2, %0;" ::"n"(32 * (kEpiWarps + 1)) : "memory");
            }
        }
    }
    ptx::tc_fence_before();
    __syncthreads();
    if (warp == kMmaWarp) ptx::tmem_dealloc(sh.tmem_base, p.tmem_cols);
    if (threadIdx.x == 0) run_exit(p.counters);
}


}  // namespace ws

// ------------------------------------------------------------------------------------------------ host
static unsigned long long *ws_trace_buf = nullptr;
static int ws_trace_cap = 0;

// Debug task trace (BDL_TRACE=<records>): 16 x u64 per task (12 used by the single-CTA kernel), read back by bdl_debug_ws_trace (tools/trace_ws.py).
unsigned long long *ws_trace_setup(unsigned char *wsp, const Subgraph &sg, cudaStream_t s, int *cap_out) {
    *cap_out = 0;
    const char *e = getenv("BDL_TRACE");
    if (!e) return nullptr;
    static unsigned long long *tbuf = nullptr;
    static int tcap = 0;
    const int cap = atoi(e);
    if (cap <= 0) return nullptr;
    if (!tbuf || cap > tcap) {
        if (tbuf) cudaFree(tbuf);
        cudaMalloc(&tbuf, (size_t)cap * 16 * 8);
        tcap = cap;
    }
    cudaMemsetAsync(tbuf, 0, (size_t)cap * 16 * 8, s);
    cudaMemsetAsync(wsp + sg.counter_off + 7 * 8, 0, 8, s);   // trace index
    ws_trace_buf = tbuf;
    ws_trace_cap = cap;
    *cap_out = cap;
    return tbuf;
}

struct WsGeom {
    int Tb, Tw, Wt, rowsA, nin, nacc, ntl, tmem_cols, smem;
};

static int ilog2(int v) {
    int r = 0;
    while ((1 << r) < v) r++;
    return (1 << r) == v ? r : -1;
}

bool ws_geometry(const bdl_plan *p, const Subgraph &sg, WsGeom &g) {
    const Layer &f = p->layers[sg.first];
    const int C = f.L.cin;
    const int H = f.in_ext[2], W = f.in_ext[3];
    const int Bh = p->in_layout.Bh, Bw = p->in_layout.Bw;
    if (p->in_layout.nsp != 2 || ilog2(Bh) < 0 || ilog2(Bw) < 0) return false;
    const bool tma = C % 64 == 0;
    const int limit = 227 * 1024 - 4096;
    const int wbytes = ws::kWS * ws::kTPS * C * C * 2;
    const int bias = (sg.last - sg.first + 1) * C * 4;
    const int Wfull = (W + Bw - 1) / Bw * Bw;
    double best = -1;
    WsGeom cand;
    // TMA path: any band height (bands need not align with bricks; a task is a Tb-row band);
    // cp.async path: one brick row per band.
    for (int Tb = tma ? std::min(H, 16) : Bh; Tb >= (tma ? 1 : Bh); Tb--) {
        for (int Tw = Wfull; Tw >= Bw; Tw -= Bw) {
            cand.Tb = Tb;
            cand.Tw = Tw;
            cand.Wt = Tw + 2;
            const int M = Tb * cand.Wt;
            cand.ntl = (M + 127) / 128;
            const int cols = cand.ntl * C;
            if (cols > 512) continue;
            cand.rowsA = (cand.ntl * 128 + 2 * cand.Wt + 2 + 7) / 8 * 8;
            if (!tma) cand.rowsA += 1;  // unswizzled chunk planes: odd 16-B stride, conflict-free cp.async stores
            const int inb = (C / 8) * cand.rowsA * 16;
            const int stage = tma ? ((C / 64) * Tb * cand.Wt * 128 + 1023) / 1024 * 1024 : 0;
            cand.nacc = 2 * cols <= 512 ? 2 : 1;
            cand.tmem_cols = 32;
            while (cand.tmem_cols < cols * cand.nacc) cand.tmem_cols *= 2;
            for (cand.nin = 2; cand.nin >= 1; cand.nin--) {
                cand.smem = inb * cand.nin + stage + wbytes + bias;
                if (cand.smem <= limit) break;
            }
            if (cand.smem > limit) continue;
            // score: useful fraction of MMA rows, double-buffered input and accumulators, then taller bands
            // (fewer tasks: per-task pipeline overheads dominate below ~3 M tiles per task; measured on B200,
            // Tb = 6 / 2 buffers beats Tb = 4 / 3 buffers at cfg2, 56 vs 62 us)
            const double eff = (double)Tb * Tw / (cand.ntl * 128.0) * (cand.nin >= 2 ? 1.0 : 0.7) *
                               (cand.nacc == 2 ? 1.0 : 0.8);
            const double score = eff + 1e-3 * Tb;
            if (score > best) {
                best = score;
                g = cand;
            }
            break;  // widest fitting Tw for this Tb
        }
    }
    if (best <= 0) return false;
    // task ids are packed as (layer << 24) | tile in the order list: the tile index must fit 24 bits
    const long long ntiles = (long long)f.in_ext[0] * ((H + g.Tb - 1) / g.Tb) * ((W + g.Tw - 1) / g.Tw);
    return ntiles < (1LL << 24);
}

// Locality-aware wavefront order (host): step s, image n, layer l -> tile row b = s - lag*l.
std::vector<int> ws_order(const bdl_plan *p, const Subgraph &sg, const WsGeom &g, int lag) {
    const Layer &f = p->layers[sg.first];
    const int L = sg.last - sg.first + 1;
    const int N = f.in_ext[0], H = f.in_ext[2], W = f.in_ext[3];
    const int nty = (H + g.Tb - 1) / g.Tb, ntx = (W + g.Tw - 1) / g.Tw;
    std::vector<int> ord;
    for (int s = 0; s < nty + lag * (L - 1); s++)
        for (int n = 0; n < N; n++)
            for (int l = 0; l < L; l++) {
                int b = s - lag * l;
                if (b < 0 || b >= nty) continue;
                for (int tx = 0; tx < ntx; tx++) ord.push_back((l << 24) | (int)(((long long)n * nty + b) * ntx + tx));
            }
    return ord;
}

// Pair kernel order: like ws_order, but per step all images of one layer are consecutive and every (step, layer)
// run is padded to an even length with -1 entries, so the two entries of a pair ticket share a layer.
std::vector<int> ws_pair_order(const bdl_plan *p, const Subgraph &sg, const WsGeom &g, int lag) {
    const Layer &f = p->layers[sg.first];
    const int L = sg.last - sg.first + 1;
    const int N = f.in_ext[0], H = f.in_ext[2];
    const int nty = (H + g.Tb - 1) / g.Tb;
    std::vector<int> ord;
    for (int s = 0; s < nty + lag * (L - 1); s++)
        for (int l = 0; l < L; l++) {
            const int b = s - lag * l;
            if (b < 0 || b >= nty) continue;
            for (int n = 0; n < N; n++) ord.push_back((l << 24) | (n * nty + b));
            if (ord.size() % 2) ord.push_back(-1);
        }
    return ord;
}

template <int C>
static bdl_status launch_ws_C(bdl_plan *p, Subgraph &sg, ws::Params &P, const WsGeom &g, bool unmerged, cudaStream_t s,
                              int *launches) {
    auto k = ws::memo_ws_kernel<C>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, g.smem);
    const long long ntiles = (long long)(P.nty) * P.ntx * p->layers[sg.first].in_ext[0];
    int grid = (int)std::min<long long>(ntiles * (unmerged ? 1 : P.L), (long long)p->num_sms);
    if (!unmerged) {
        P.only_layer = -1;
        launch_pdl(k, dim3(grid), dim3(ws::Roles<C>::THREADS), g.smem, s, P);
        *launches += 1;
    } else {
        P.order = nullptr;
        P.norder = ntiles;
        grid = (int)std::min<long long>(ntiles, (long long)p->num_sms);
        for (int l = 0; l < P.L; l++) {
            P.only_layer = l;
            launch_pdl(k, dim3(grid), dim3(ws::Roles<C>::THREADS), g.smem, s, P);
            *launches += 1;
        }
    }
    BDL_CUDA_CHECK_LAUNCH("tcgen05 memo ws kernel");
    return BDL_OK;
}

bdl_status launch_tc_subgraph(bdl_plan *p, Subgraph &sg, const TView &in, const TView &out, const TView *res,
                              unsigned char *ws, cudaStream_t s, int *launches);

// TMA descriptor of a bricked bf16 tensor viewed as 2-D [pixels][Cp]: box = 64 channels x box_px pixels,
// 128-B swizzle (matches the UMMA SWIZZLE_128B A-operand layout).
static bool encode_pixel_map(CUtensorMap *tm, const TView &v, int box_px) {
    static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult qr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &qr) != cudaSuccess ||
            !enc)
            return false;
    }
    long long nbricks = (long long)v.nb[0] * v.nb[1] * v.nb[2] * v.nb[3];
    cuuint64_t dims[2] = {(cuuint64_t)v.Cp, (cuuint64_t)(nbricks * (v.brick_elems / v.Cp))};
    cuuint64_t strides[1] = {(cuuint64_t)v.Cp * 2};
    cuuint32_t box[2] = {64, (cuuint32_t)box_px};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, v.ptr, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// 5-D view of a 2-D bricked bf16 tensor (identity BrickMap): (channel, x in brick, brick column,
// y in brick, brick row over (n, by)); box = 64 channels x Bw x nseg bricks x 1 x 1 = one tile row.
static bool encode_row_map(CUtensorMap *tm, const TView &v, int nseg, int rows = 1);
// Like encode_row_map with a box of `rows` pixel rows of one brick row; nseg may exceed the bricks per row (the
// boxes' extra bricks read outside the map: zero fill).
bool encode_rows_map_bf16(CUtensorMap *tm, const TView &v, int nseg, int rows) { return encode_row_map(tm, v, nseg, rows); }
static bool encode_row_map(CUtensorMap *tm, const TView &v, int nseg, int rows) {
    static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult qr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &qr) != cudaSuccess ||
            !enc)
            return false;
    }
    const cuuint64_t px = (cuuint64_t)v.Cp * 2, brick = (cuuint64_t)v.brick_elems * 2;
    cuuint64_t dims[5] = {(cuuint64_t)v.Cp, (cuuint64_t)v.B[3], (cuuint64_t)v.nb[3], (cuuint64_t)v.B[2],
                          (cuuint64_t)v.nb[0] * v.nb[1] * v.nb[2]};
    cuuint64_t strides[4] = {px, brick, px * v.B[3], brick * v.nb[3]};
    cuuint32_t box[5] = {64, (cuuint32_t)v.B[3], (cuuint32_t)nseg, (cuuint32_t)rows, 1};
    cuuint32_t es[5] = {1, 1, 1, 1, 1};
    CUresult r = enc(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, v.ptr, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

bool encode_row_map_bf16(CUtensorMap *tm, const TView &v, int nseg) { return encode_row_map(tm, v, nseg); }

bool pair_geometry(int L, int H, int W, int Bw, int N, int num_sms, int &Tb, int &ntl, int &in_bytes, int &smem, int &nin);
bdl_status launch_pair_subgraph(const bdl_plan *p, const Subgraph &sg, const TView &in, const TView &out, const TView *res,
                                unsigned char *wsp, cudaStream_t s, int *launches, bool unmerged, void *dense);

// The CTA-pair kernel (chain_tc_pair.cu) runs C = 64 chains over full-width bands when their weights fit resident;
// returns its band height, or 0.  BDL_NO_PAIR=1 keeps the single-CTA kernel (A/B runs).
int pair_band_rows(const bdl_plan *p, const Subgraph &sg) {
    const char *np = getenv("BDL_NO_PAIR");
    const bool off = np && atoi(np);
    const Layer &f = p->layers[sg.first];
    if (off || f.L.cin != 64 || p->in_layout.nsp != 2 || p->in_layout.brickmap || p->in_layout.Bh > 8) return 0;
    if (ilog2(p->in_layout.Bh) < 0 || ilog2(p->in_layout.Bw) < 0) return 0;
    int Tb, ntl, ib, sm, nin;
    if (!pair_geometry(sg.last - sg.first + 1, f.in_ext[2], f.in_ext[3], p->in_layout.Bw, f.in_ext[0], p->num_sms, Tb, ntl,
                       ib, sm, nin))
        return 0;
    return Tb;
}

bdl_status launch_ws_subgraph(bdl_plan *p, Subgraph &sg, const TView &in, const TView &out, const TView *res,
                              unsigned char *wsp, cudaStream_t s, int *launches, bool unmerged, void *dense) {
    if (pair_band_rows(p, sg) > 0 && !in.bmap && !out.bmap && !(res && res->bmap))
        return launch_pair_subgraph(p, sg, in, out, res, wsp, s, launches, unmerged, dense);
    WsGeom g;
    if (!ws_geometry(p, sg, g)) return fail(BDL_EUNSUPPORTED, "tcgen05 ws kernel: tile does not fit on chip");
    ws::Params P;
    memset(&P, 0, sizeof(P));
    P.dense = (__nv_bfloat16 *)dense;
    const Layer &f = p->layers[sg.first];
    const int L = sg.last - sg.first + 1;
    P.L = L;
    P.C = f.L.cin;
    P.H = f.in_ext[2];
    P.W = f.in_ext[3];
    P.Tb = g.Tb;
    P.Tw = g.Tw;
    P.Wt = g.Wt;
    P.nty = (P.H + g.Tb - 1) / g.Tb;
    P.ntx = (P.W + g.Tw - 1) / g.Tw;
    P.lBh = ilog2(p->in_layout.Bh);
    P.lBw = ilog2(p->in_layout.Bw);
    P.rowsA = g.rowsA;
    P.stage_off = (P.C / 8) * g.rowsA * 16 * g.nin;
    P.nin = g.nin;
    P.nacc = g.nacc;
    P.ntl = g.ntl;
    P.tmem_cols = g.tmem_cols;
    P.in = in;
    if (res) P.res = *res;
    for (int j = 0; j < L; j++) {
        const Layer &ly = p->layers[sg.first + j];
        ws::Layer &T = P.layer[j];
        T.w = (const __nv_bfloat16 *)(wsp + ly.tc_w_off);
        T.bias = (const float *)(wsp + ly.b_off);
        T.relu = ly.L.relu;
        T.res = sg.res_tensor[j] >= 0;
        if (j == L - 1) {
            T.out = out;
        } else {
            bdl_layout lo;
            bdl_layout_init(&lo, 2, ly.out_ext[0], ly.L.cout, 1, ly.out_ext[2], ly.out_ext[3], p->in_layout.Bn, 1,
                            p->in_layout.Bh, p->in_layout.Bw, BDL_BF16);
            T.out = make_view(lo, wsp + sg.memo_off[j]);
        }
        P.task_base[j] = sg.task_base[j];
    }
    if (P.C % 64 == 0) {
        if (in.bmap || out.bmap || (res && res->bmap))  // the TMA epilogue needs consecutive bricks per row (planner)
            return fail(BDL_EUNSUPPORTED, "tcgen05 ws kernel: a BrickMap needs the generic kernel");
        P.row_tma = 1;
        for (int j = 0; j < L; j++)
            if (!encode_row_map(&P.tm_out[j], P.layer[j].out, g.Tw >> P.lBw))
                return fail(BDL_ECUDA, "cuTensorMapEncodeTiled (output row map) failed");
        if (res && !encode_row_map(&P.tm_res, *res, g.Tw >> P.lBw))
            return fail(BDL_ECUDA, "cuTensorMapEncodeTiled (residual row map) failed");
        for (int j = 0; j < L; j++) {
            const TView &src = j == 0 ? P.in : P.layer[j - 1].out;
            if (!encode_pixel_map(&P.tm_seg[j], src, 1 << P.lBw))
                return fail(BDL_ECUDA, "cuTensorMapEncodeTiled failed for a brick tensor");
            if (P.row_tma && !encode_row_map(&P.tm_row[j], src, g.Tw >> P.lBw))
                return fail(BDL_ECUDA, "cuTensorMapEncodeTiled (5-D row map) failed");
        }
    }
    P.status = (int *)(wsp + sg.status_off);
    P.counters = (unsigned long long *)(wsp + sg.counter_off);
    P.order = sg.order_off >= 0 ? (const int *)(wsp + sg.order_off) : nullptr;
    P.norder = sg.norder;
#ifdef BDL_DEBUG   // timing knobs that deliberately skip work (wrong results): debug builds only
    if (const char *e = getenv("BDL_WS_DBG")) P.dbg = atoi(e);
#endif
    P.trace = ws_trace_setup(wsp, sg, s, &P.trace_cap);
    switch (P.C) {
        case 16: return launch_ws_C<16>(p, sg, P, g, unmerged, s, launches);
        case 32: return launch_ws_C<32>(p, sg, P, g, unmerged, s, launches);
        case 64: return launch_ws_C<64>(p, sg, P, g, unmerged, s, launches);
        case 128: return launch_ws_C<128>(p, sg, P, g, unmerged, s, launches);
    }
    return fail(BDL_EUNSUPPORTED, "tcgen05 ws kernel: channel count");
}

}  // namespace bdl

namespace bdl {
std::vector<int> ws_task_order(const bdl_plan *p, const Subgraph &sg) {
    WsGeom g;
    if (!ws_geometry(p, sg, g)) return {};
    const bool pair = pair_band_rows(p, sg) > 0;
    if (pair) {
        g.Tb = pair_band_rows(p, sg);
        g.Tw = p->layers[sg.first].in_ext[3];
    }
    // lag: how many band rows layer l trails layer l-1.  Larger = fewer dependency waits but a larger
    // live intermediate; take the largest lag whose live intermediate (lag band rows of every image of
    // the shard, per merged layer) fits in a quarter of L2, at least 3.
    const Layer &f = p->layers[sg.first];
    const int L = sg.last - sg.first + 1;
    const int nty = (f.in_ext[2] + g.Tb - 1) / g.Tb;
    const double band_bytes = (double)f.in_ext[0] * g.Tb * f.in_ext[3] * f.L.cin * 2.0;
    int lag = (int)std::min<double>(nty, (double)p->l2_bytes / 4.0 / std::max(1, L - 1) / band_bytes);
    lag = std::max(3, lag);
    if (const char *e = getenv("BDL_LAG")) lag = std::max(1, atoi(e));
    std::vector<int> ord = pair ? ws_pair_order(p, sg, g, lag) : ws_order(p, sg, g, lag);
    if (p->opts.schedule_seed) {  // any order is valid: the scheduler claims missing dependencies first
        std::mt19937 rng((unsigned)p->opts.schedule_seed);
        std::shuffle(ord.begin(), ord.end(), rng);
    }
    return ord;
}
}  // namespace bdl

extern "C" int32_t bdl_plan_subgraph_cta_pair(const bdl_plan *p, int32_t i) {
    if (!p || i < 0 || i >= (int)p->sgs.size()) return 0;
    const bdl::Subgraph &sg = p->sgs[i];
    return bdl::effective_kernel(sg) == bdl::KERNEL_TC_BAND && bdl::pair_band_rows(p, sg) > 0 ? 1 : 0;
}

// Debug: copy the warp-specialized kernel's task trace (8 x u64 per task) to host.
extern "C" int bdl_debug_ws_trace(unsigned long long *host, int max_records) {
    if (!bdl::ws_trace_buf) return 0;
    int n = max_records < bdl::ws_trace_cap ? max_records : bdl::ws_trace_cap;
    cudaDeviceSynchronize();
    cudaMemcpy(host, bdl::ws_trace_buf, (size_t)n * 16 * 8, cudaMemcpyDeviceToHost);
    return n;
}

namespace bdl {
// Band height of the warp-specialized kernel for subgraph sg (0 if it cannot run it).
int pair_band_rows(const bdl_plan *p, const Subgraph &sg);
int ws_band_rows(const bdl_plan *p, const Subgraph &sg) {
    if (int tb = pair_band_rows(p, sg)) return tb;
    WsGeom g;
    return ws_geometry(p, sg, g) ? g.Tb : 0;
}
}  // namespace bdl
