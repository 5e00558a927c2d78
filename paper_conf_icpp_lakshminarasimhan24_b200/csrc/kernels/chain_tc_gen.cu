// Generic warp-specialized tcgen05 kernel for MEMOIZED and UNMERGED execution of conv chains of any
// shape the paper's workloads use (§3.2.2 Fig 2d, §4.3-§4.5): 2-D and 3-D, kernel sizes up to
// 7, stride 1 or 2, any channel counts (cin <= 8, multiples of 16, multiples of 64), cin != cout,
// bias / residual / ReLU epilogues.  The C = 64/128 3x3 chain of the bench config has its own tuned
// kernel (chain_tc_ws.cu); this one covers everything else on the tensor cores.
//
// Implicit GEMM over an output TILE (Tb rows x Tw columns of one output plane, one chunk of Nc output
// channels): M = 128 flattened tile positions m = i*Wp + j, N = Nc, K = input channels x taps.  The input
// tile is staged in shared memory as pixel rows such that every tap (a, r, s) is a constant row offset
// ("shifted window"): for stride 2 the tile is stored as polyphase blocks (row parity x column parity),
// so a tap's rows are again contiguous.  Channels stream through the K loop in K-blocks (64 channels =
// one 128-B swizzled pixel row); taps x 16-channel k-steps of each K-block are MMAs with a per-layer
// table of A-descriptor offsets.  cin <= 8 (the RGB stem layers) packs two taps into one K = 16 step
// through the descriptor's leading-byte offset.
//
// Roles (one CTA per SM, persistent):
//   warp 0       scheduler: ticket counter over a topological (image-group, layer) order, CAS claims
//                (0 -> 1, L513-531), claims not-started dependencies first (Fig 2d recursion)
//   warps 1-4    loaders: wait for the dependency tiles (state 2), cp.async the K-blocks of the input
//                tile into an input-stage ring (zero-fill outside the image)
//   warp 5       weight producer: bulk copies of packed weight stages into a ring
//   warp 6       MMA issuer (warp-converged, elected lane issues)
//   warps 7-22   epilogue: tcgen05.ld -> +bias (+residual) -> ReLU -> bf16 -> bricked global stores,
//                then release-publish the tile (state 2)
#include <algorithm>
#include <cstdio>
#include <cmath>
#include <random>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "common.cuh"
#include "tc_ptx.cuh"

namespace bdl {

namespace gen {

// Warp roles; the epilogue has EPIW warps (a template parameter: 8 or 12, EPIW / 4 per TMEM lane quadrant).  Fewer
// warps leave more registers per thread (19 warps: 96, 15 warps: 128; 23 warps were capped at 80 and spilled).
constexpr int kSched = 0, kLoad0 = 1, kLW = 4, kWProd = 5, kMma = 6, kEpi0 = 7;
constexpr int kLoadT = 32 * kLW;
constexpr int kQ = 4, kRing = 16, kStack = 128;
constexpr int kPendDraw = 32, kPend = kPendDraw + kStack;   // pending (deferred) tasks: draw tickets below kPendDraw
constexpr int kMaxIn = 4, kMaxW = 4, kMaxKs = 128;   // k-steps per layer: 3x3x3 taps x 64 channels = 108
constexpr int kTaskBits = 26;   // order entry = (layer << kTaskBits) | task

enum { AM_SW128 = 0, AM_PLANES = 1, AM_PAIR = 2, AM_SW64 = 3 };   // AM_SW64: cin = 32, 64-B swizzled pixel rows

struct LayerP {
    TView src, out, res;
    const __nv_bfloat16 *w;   // packed [nc][kb][ks][2][Nc][8]
    int srcl, resl;           // producer (index in the subgraph) of the input / of the residual, -1 = external
    // fused max-pool (the subgraph ends in a pool of this conv, L620-626): the task grid and `out` are the POOLED
    // output; a task is a Tpb x Tpw tile of pool outputs and computes the conv tile under its windows
    // (Tb = (Tpb-1)*ps + pk rows, Fig 4 rule with the pool's stride as padding factor, L456-458), pools it in
    // the epilogue and never materializes the conv output
    int pool;
    int pk[2], ps[2], ppd[2]; // pool window / stride / padding (h, w)
    int pout[3];              // pooled output extents (d, h, w); out_ext stays the conv's
    int Tpb, Tpw;
    const float *bias;        // [cout]
    int bofs;                 // float offset of this layer's bias in the shared bias table (Params::bias_off)
    int relu, has_res;
    int cin, cout;
    int k[3], s[3], pd[3];    // (d, h, w)
    int dl[3], ke[3];         // dilation; window input extent ke = dl*(k-1) + 1 (dilated convs: SURVEY Q19)
    int stk, Td;              // depth stacking (3-D, k0 = 3): a task computes Td output planes and one MMA of N = up to
                              // 3 Nc feeds up to three of them from one input plane (stk = 0: Td = 1)
    uint32_t idesc_s[3];      // stacked MMAs: instruction descriptors for N = Nc, 2 Nc, 3 Nc
    int in_ext[3], out_ext[3];
    int grid[3];              // output bricked-grid extents (D, H, W)
    int Tb, Tw, Wp;
    int ntd, nty, ntx, nnc, Nc;
    int amode, nkb, kc, nks, kpw, nws;   // kc: 16-B chunks per pixel per K-block
    int lkc;                  // log2(kc)
    int tma;                  // 1: the in-image columns of each input row arrive by one TMA box (tm_row)
    int pxo;                  // SW64: pixel-row offset of the stage (0/1) that makes every TMA row start 128-B aligned
    int xal;                  // padded mode, first layer: tiles start at the region's x rounded down to a brick
                              // boundary, so their in-tile columns are whole brick-row segments (TMA boxes)
    int lB[3];                // log2 of the source view's brick extents (d, h, w)
    int rb, nblk, blk_px, plane_px;
    int in_rows, in_cols;
    int rowsA, stage_bytes, row_u;       // row_u: 16-B units per A row (8 swizzled, 1 planes)
    int ntl;
    uint32_t idesc;
    long long task_base, ntasks;
    int pR[3];                // padded: largest region of this layer's output (scratch pitches)
    long long scr_off;        // padded: byte offset of the layer's region buffer in a scratch slot
    int l2hint;               // epilogue stores' L2 policy: 1 evict_last (a later layer of the subgraph reads this
                              // output: keep it resident), 2 evict_first (leaves the subgraph: stream it), 0 none
};

struct Params {
    CUtensorMap tm_row[kMaxLayers];      // 5-D row map of each layer's source (LayerP::tma): box = Tw pixels x 64 ch
    LayerP layer[kMaxLayers];
    int L;
    int nin, nw, in_stride, w_stride;    // ring depths and slot strides (bytes)
    int pool_off;                        // fused pool: byte offset of the epilogue staging tile in dynamic smem
    int bias_off;                        // byte offset of the fp32 bias table (every layer's cout) in dynamic smem, or
                                         // -1: the epilogue then reads each item's biases by one global load + shuffles
    int nacc, acc_stride, tmem_cols;
    int *status;
    int defer;                           // bdl_plan_opts.memo_defer: 1 = hand over only ready tasks (revisit the others)
    unsigned long long *counters;        // run state (common.cuh run_epoch / run_exit)
    const int *order;                    // (l << 26) | task, or null (unmerged)
    long long norder;
    int only_layer;
    // padded mode (§3.2.1): a task is a PB block of the last layer's output; every layer's
    // halo-extended region is recomputed by the CTA into its private scratch (two slots, so two blocks
    // interleave and one block's loads overlap the other's MMAs)
    int dbg;                             // debug timing knobs (BDL_GEN_DBG): 1 = one k-step per task, 2 = no input loads,
                                         // 4 = no epilogue stores, 8 = no bias reads, 16 = no residual reads (all give
                                         // wrong results)
    unsigned long long *prof;            // debug (BDL_GEN_PROF): per CTA 32 x u64 of role wait / busy cycles, or null
    int padded;
    int PB[3], npb[3];
    unsigned char *scratch;
    long long scr_slot;
};

struct Shared {
    uint64_t q_full[kQ], q_empty[kQ];
    uint64_t in_full[kMaxIn], in_empty[kMaxIn], wfull[kMaxW], wempty[kMaxW];
    uint64_t acc_full[2], acc_empty[2];
    uint64_t desc_full[kRing];
    uint32_t tmem_base;
    int q_l[kQ], q_w[kQ];                // q_w: padded: sub-task seq whose epilogue must be done first
    long long q_t[kQ];
    int done_seq;                        // padded: sub-tasks whose epilogue stores are complete
    int desc_l[kRing];
    long long desc_t[kRing];
    int stk_l[kStack];
    long long stk_t[kStack];
    int pend_l[kPend];
    long long pend_t[kPend];
    uint32_t ks[kMaxLayers][kMaxKs];     // per k-step: A offset | LBO << 16 (both in 16-B units, < 2^14)
};

// detailed per-phase timers of the debug profiler (BDL_GEN_PROF): debug builds only (they cost the release kernel
// registers and issue slots)
#ifdef BDL_DEBUG
#define PT(x) x
#define DBG(p, bit) ((p).dbg & (bit))   // work-skipping timing knobs (wrong results)
#else
#define PT(x)
#define DBG(p, bit) 0
#endif
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ptx::smem_u32(bar)) : "memory");
}
// debug profiler: time spent blocked in an mbarrier wait (only when p.prof is set)
__device__ __forceinline__ void pwait(const Params &p, uint64_t *bar, uint32_t parity, unsigned long long &acc) {
    if (p.prof) {
        const unsigned long long t0 = clock64();
        ptx::mbar_wait(bar, parity);
        acc += clock64() - t0;
    } else {
        ptx::mbar_wait(bar, parity);
    }
}
__device__ __forceinline__ int tag_state(int v, unsigned EP) { return ((v & ~1023) == (int)EP) ? (v & 3) : 0; }
__device__ __forceinline__ int *status_word(const Params &p, int l, long long t) {
    return p.status + p.layer[l].task_base + t;
}

// K-step q of a layer whose A layout is not tap-paired: the depth tap is the FASTEST index, q = (rs * kpt + kk) * k0 + a
// (rs = r * k2 + s, kk = 16-channel slice of the K-block).  Every output element then accumulates, per (r, s, kk),
// the depth taps a = 0, 1, 2 in order -- the order the depth-stacked MMAs of 3-D layers produce (one MMA feeds three
// output planes from one input plane), so stacked and unstacked execution of a layer give the same bits.
__host__ __device__ __forceinline__ void kstep_tap(int q, int k0, int k1, int k2, int kpt, int &tap, int &kk) {
    const int a = q % k0;
    q /= k0;
    kk = q % kpt;
    const int rs = q / kpt;
    tap = (a * k1 + rs / k2) * k2 + rs % k2;
}

struct TaskC { int n, d, ty, tx, nc; };
// (task ids fit 32 bits, kTaskBits: 32-bit unsigned divisions, several times cheaper than 64-bit ones on the
// per-task path of the scheduler, loaders and epilogue)
__host__ __device__ __forceinline__ TaskC decode(const LayerP &L, long long t64) {
    TaskC c;
    unsigned t = (unsigned)t64, q;
    q = t / (unsigned)L.nnc; c.nc = (int)(t - q * (unsigned)L.nnc); t = q;
    q = t / (unsigned)L.ntx; c.tx = (int)(t - q * (unsigned)L.ntx); t = q;
    q = t / (unsigned)L.nty; c.ty = (int)(t - q * (unsigned)L.nty); t = q;
    q = t / (unsigned)L.ntd; c.d = (int)(t - q * (unsigned)L.ntd);
    c.n = (int)q;
    return c;
}

// Element offset of channel 0 of pixel (n, d, y, x) in a bricked view (Bn = 1), power-of-two bricks
// with log2 extents lB (d, h, w).
__device__ __forceinline__ long long pix_pow2(const TView &v, const int *lB, int n, int d, int y, int x) {
    const int bd = d >> lB[0], by = y >> lB[1], bx = x >> lB[2];
    const long long logical = (((long long)n * v.nb[1] + bd) * v.nb[2] + by) * v.nb[3] + bx;
    const long long phys = v.bmap ? (long long)v.bmap[logical] : logical;
    const int in = ((((d - (bd << lB[0])) << lB[1]) + (y - (by << lB[1]))) << lB[2]) + (x - (bx << lB[2]));
    return phys * v.brick_elems + (long long)in * v.Cp;
}

// Element offset of channel 0 of pixel (n, d, y, x) in a bricked view (Bn = 1).
__device__ __forceinline__ long long pix(const TView &v, int n, int d, int y, int x) {
    const int bd = d / v.B[1], by = y / v.B[2], bx = x / v.B[3];
    const long long logical = (((long long)n * v.nb[1] + bd) * v.nb[2] + by) * v.nb[3] + bx;
    const long long phys = v.bmap ? (long long)v.bmap[logical] : logical;
    const int in = (((d - bd * v.B[1]) * v.B[2]) + (y - by * v.B[2])) * v.B[3] + (x - bx * v.B[3]);
    return phys * v.brick_elems + (long long)in * v.Cp;
}

// First conv-output row / column of tile (ty, tx) (pooled layers: under its first pool window; may be < 0).
// Fused pool: channel batches staged together in the epilogue -- a power of two (the staging tile's XOR swizzle
// masks with the chunk count), <= 4 / M tiles so the 4 warp ranks share ntl x gcb items
__host__ __device__ __forceinline__ int pool_gcb(int ncb, int ntl, int er) {
    int g = ncb < er / ntl ? ncb : er / ntl;
    if (g < 1) g = 1;
    while (g & (g - 1)) g &= g - 1;
    return g;
}
__host__ __device__ __forceinline__ int tile_y0(const LayerP &L, int ty) {
    return L.pool ? ty * L.Tpb * L.ps[0] - L.ppd[0] : ty * L.Tb;
}
__host__ __device__ __forceinline__ int tile_x0(const LayerP &L, int tx) {
    return L.pool ? tx * L.Tpw * L.ps[1] - L.ppd[1] : tx * L.Tw;
}

// Dependencies of task t of layer C: the tiles of its input producer P covering its input window (every channel
// chunk of P), and the tiles of its residual producer R covering its output tile (the same channel chunk).
struct DepRange { int n, d0, nd, b0, nb, x0, nx, c0, nnc; };
__host__ __device__ __forceinline__ DepRange dep_range_src(const LayerP &C, const LayerP &P, long long t) {
    const TaskC c = decode(C, t);
    DepRange r;
    r.n = c.n;
    r.c0 = 0;
    r.nnc = P.nnc;
    int lo, hi;
    // (tasks of depth-stacked layers cover Td planes: C's planes [c.d*Td, +Td), P's blocks of P.Td planes)
    lo = max(0, c.d * C.Td * C.s[0] - C.pd[0]);
    hi = min(C.in_ext[0] - 1, (c.d * C.Td + C.Td - 1) * C.s[0] - C.pd[0] + C.ke[0] - 1);
    if (P.Td == 1) {   // (2-D and unstacked layers: no division on the per-task path)
        r.d0 = lo;
        r.nd = max(0, hi - lo + 1);
    } else {
        r.d0 = lo / P.Td;
        r.nd = hi >= lo ? hi / P.Td - r.d0 + 1 : 0;
    }
    const int y0 = tile_y0(C, c.ty), x0 = tile_x0(C, c.tx);
    lo = max(0, y0 * C.s[1] - C.pd[1]);
    hi = min(C.in_ext[1] - 1, (y0 + C.Tb - 1) * C.s[1] - C.pd[1] + C.ke[1] - 1);
    r.b0 = lo / P.Tb;
    r.nb = hi >= lo ? hi / P.Tb - r.b0 + 1 : 0;
    lo = max(0, x0 * C.s[2] - C.pd[2]);
    hi = min(C.in_ext[2] - 1, (x0 + C.Tw - 1) * C.s[2] - C.pd[2] + C.ke[2] - 1);
    r.x0 = lo / P.Tw;
    r.nx = hi >= lo ? hi / P.Tw - r.x0 + 1 : 0;
    return r;
}
__host__ __device__ __forceinline__ DepRange dep_range_res(const LayerP &C, const LayerP &R, long long t) {
    const TaskC c = decode(C, t);
    DepRange r;
    r.n = c.n;
    r.c0 = c.nc;     // same cout, same Nc: the same channel chunk
    r.nnc = 1;
    {
        const int dlo = c.d * C.Td, dhi = min(C.out_ext[0], dlo + C.Td) - 1;
        r.d0 = R.Td == 1 ? dlo : dlo / R.Td;
        r.nd = dhi >= dlo ? (R.Td == 1 ? dhi : dhi / R.Td) - r.d0 + 1 : 0;
    }
    int lo = c.ty * C.Tb, hi = min(C.out_ext[1], lo + C.Tb) - 1;
    r.b0 = lo / R.Tb;
    r.nb = hi >= lo ? hi / R.Tb - r.b0 + 1 : 0;
    lo = c.tx * C.Tw;
    hi = min(C.out_ext[2], lo + C.Tw) - 1;
    r.x0 = lo / R.Tw;
    r.nx = hi >= lo ? hi / R.Tw - r.x0 + 1 : 0;
    return r;
}
__host__ __device__ __forceinline__ int dep_count(const DepRange &r) { return r.nd * r.nb * r.nx * r.nnc; }
__host__ __device__ __forceinline__ long long dep_task(const LayerP &P, const DepRange &r, int i) {
    unsigned u = (unsigned)i, q;
    q = u / (unsigned)r.nnc; const int c = r.c0 + (int)(u - q * (unsigned)r.nnc); u = q;
    q = u / (unsigned)r.nx; const int x = r.x0 + (int)(u - q * (unsigned)r.nx); u = q;
    q = u / (unsigned)r.nb; const int b = r.b0 + (int)(u - q * (unsigned)r.nb);
    const int d = r.d0 + (int)q;
    return (long long)(((((unsigned)r.n * P.ntd + d) * P.nty + b) * P.ntx + x) * P.nnc + c);
}
// All dependencies of (l, t) as one index space: [0, ns) on the input producer, [ns, ns + nr) on the residual's.
struct Deps {
    DepRange s, r;
    int ns, nr, ls, lr;
};
__host__ __device__ __forceinline__ Deps deps_of(const LayerP *ly, int l, long long t) {
    Deps D;
    const LayerP &C = ly[l];
    D.ls = C.srcl;
    D.lr = C.resl;
    D.ns = D.nr = 0;
    if (C.srcl >= 0) {
        D.s = dep_range_src(C, ly[C.srcl], t);
        D.ns = dep_count(D.s);
    }
    if (C.resl >= 0) {
        D.r = dep_range_res(C, ly[C.resl], t);
        D.nr = dep_count(D.r);
    }
    return D;
}
// i-th dependency: its layer and task
__host__ __device__ __forceinline__ long long dep_at(const LayerP *ly, const Deps &D, int i, int &dl) {
    if (i < D.ns) {
        dl = D.ls;
        return dep_task(ly[D.ls], D.s, i);
    }
    dl = D.lr;
    return dep_task(ly[D.lr], D.r, i - D.ns);
}

// Padded mode: region of layer l's output needed for block (bd, by, bx) of the last layer (Fig 4:
// reverse traversal, input extent s*(O-1) + k, clipped to the feature map).  lo/hi: [lo, hi) per dim.
__host__ __device__ inline void region_of(const LayerP *ly, int L, const int PB[3], const int blk[3], int l, int lo[3],
                                          int hi[3]) {
    for (int d = 0; d < 3; d++) {
        lo[d] = blk[d] * PB[d];
        hi[d] = lo[d] + PB[d] < ly[L - 1].grid[d] ? lo[d] + PB[d] : ly[L - 1].grid[d];
    }
    for (int j = L - 1; j > l; j--) {
        const LayerP &J = ly[j];
        if (J.pool) {   // pooled output region -> the conv output region under its windows (clipped to the map)
            for (int d = 1; d < 3; d++) {
                const int h = hi[d] < J.pout[d] ? hi[d] : J.pout[d];
                if (h <= lo[d]) {
                    lo[d] = hi[d] = 0;
                    continue;
                }
                const int nlo = lo[d] * J.ps[d - 1] - J.ppd[d - 1], nhi = (h - 1) * J.ps[d - 1] - J.ppd[d - 1] + J.pk[d - 1];
                lo[d] = nlo > 0 ? nlo : 0;
                hi[d] = nhi < J.out_ext[d] ? nhi : J.out_ext[d];
                if (hi[d] < lo[d]) hi[d] = lo[d];
            }
        }
        for (int d = 0; d < 3; d++) {
            const int h = hi[d] < J.out_ext[d] ? hi[d] : J.out_ext[d];
            if (h <= lo[d]) {
                lo[d] = hi[d] = 0;
                continue;
            }
            const int nlo = lo[d] * J.s[d] - J.pd[d], nhi = (h - 1) * J.s[d] - J.pd[d] + J.ke[d];
            lo[d] = nlo > 0 ? nlo : 0;
            hi[d] = nhi < J.in_ext[d] ? nhi : J.in_ext[d];
            if (hi[d] < lo[d]) hi[d] = lo[d];
        }
    }
}
// first tile column of a padded-mode region (aligned down to a brick edge for xal layers)
__host__ __device__ inline int region_x0(const LayerP &L, int lo2) {
    return L.xal ? (lo2 >> L.lB[2]) << L.lB[2] : lo2;
}
__host__ __device__ inline int region_subtiles(const LayerP &L, const int lo[3], const int hi[3]) {
    const int a = hi[0] - lo[0], b = hi[1] - lo[1], c = hi[2] - region_x0(L, lo[2]);
    if (a <= 0 || b <= 0 || c <= 0) return 0;
    const int tb = L.pool ? L.Tpb : L.Tb, tw = L.pool ? L.Tpw : L.Tw;   // pooled: tiles of the pooled region
    return a * ((b + tb - 1) / tb) * ((c + tw - 1) / tw) * L.nnc;
}

// One unit of work of the pipeline: an output tile of layer l (memoized/unmerged: a tile of the bricked
// grid; padded: a tile of a block's region), with where its input comes from and its output goes.
struct Tile {
    int n, d, y0, x0, nc;
    int py0, px0;              // pooled layers: first pool-output row / column of the tile
    int hi[3];                 // exclusive bounds of the positions this tile writes
    int src_scr, dst_scr;      // padded: input / output in the CTA's scratch
    int slo[3], shi[3];        // source region (scratch) bounds
    int dlo[3];                // destination region origin (scratch)
    int slot;
};
__device__ __forceinline__ Tile make_tile(const Params &p, int l, long long t) {
    const LayerP &L = p.layer[l];
    Tile T;
    if (!p.padded) {
        const TaskC c = decode(L, t);
        T.n = c.n; T.d = c.d * L.Td; T.y0 = tile_y0(L, c.ty); T.x0 = tile_x0(L, c.tx); T.nc = c.nc;
        T.py0 = c.ty * L.Tpb; T.px0 = c.tx * L.Tpw;
        T.hi[0] = L.grid[0]; T.hi[1] = L.grid[1]; T.hi[2] = L.grid[2];
        T.src_scr = T.dst_scr = 0;
        T.slot = 0;
        return T;
    }
    // t = ((P << 16 | k) << 8 | nc) << 1 | slot
    T.slot = (int)(t & 1);
    T.nc = (int)((t >> 1) & 0xFF);
    int k = (int)((t >> 9) & 0xFFFF);
    unsigned P = (unsigned)(t >> 25), q;
    int blk[3];
    q = P / (unsigned)p.npb[2]; blk[2] = (int)(P - q * (unsigned)p.npb[2]); P = q;
    q = P / (unsigned)p.npb[1]; blk[1] = (int)(P - q * (unsigned)p.npb[1]); P = q;
    q = P / (unsigned)p.npb[0]; blk[0] = (int)(P - q * (unsigned)p.npb[0]);
    T.n = (int)q;
    int lo[3], hi[3];
    region_of(p.layer, p.L, p.PB, blk, l, lo, hi);
    const int xs = region_x0(L, lo[2]);
    const int tb = L.pool ? L.Tpb : L.Tb, tw = L.pool ? L.Tpw : L.Tw;
    const int nty = (hi[1] - lo[1] + tb - 1) / tb, ntx = (hi[2] - xs + tw - 1) / tw;
    const int kx = k % ntx; k /= ntx;
    const int ky = k % nty;
    const int kd = k / nty;
    T.d = lo[0] + kd; T.y0 = lo[1] + ky * L.Tb; T.x0 = xs + kx * L.Tw;
    if (L.pool) {   // (lo, hi) is a pooled region
        T.py0 = lo[1] + ky * L.Tpb;
        T.px0 = xs + kx * L.Tpw;
        T.y0 = T.py0 * L.ps[0] - L.ppd[0];
        T.x0 = T.px0 * L.ps[1] - L.ppd[1];
    }
    for (int d = 0; d < 3; d++) { T.hi[d] = hi[d]; T.dlo[d] = lo[d]; }
    T.dst_scr = l < p.L - 1;
    T.src_scr = l > 0;
    if (T.src_scr) region_of(p.layer, p.L, p.PB, blk, l - 1, T.slo, T.shi);
    return T;
}
__device__ __forceinline__ unsigned char *scr_slot(const Params &p, int slot) {
    return p.scratch + ((long long)blockIdx.x * 2 + slot) * p.scr_slot;
}

// ---------------------------------------------------------------------------------------------- scheduler
__device__ void scheduler_padded(const Params &p, Shared &sh) {
    const int lane = threadIdx.x % 32;
    uint32_t qseq = 0;
    auto emit = [&](int l, long long t, int wait) {
        const int slot = qseq % kQ;
        if (qseq >= (uint32_t)kQ) ptx::mbar_wait(&sh.q_empty[slot], ((qseq / kQ) - 1) & 1);
        if (lane == 0) {
            sh.q_l[slot] = l;
            sh.q_t[slot] = t;
            sh.q_w[slot] = wait;
            mbar_arrive(&sh.q_full[slot]);
        }
        __syncwarp();
        qseq++;
    };
    unsigned long long computed = 0;
    for (;;) {
        // two blocks at a time: their layers interleave (A.l0, B.l0, A.l1, B.l1, ...) so that a layer's
        // loads wait for the previous layer of the same block while the other block's MMAs run
        // one ticket draw per pair
        long long P[2];
        int np = 0;
        unsigned long long tk = 0;
        if (lane == 0) tk = atomicAdd(&p.counters[4], 2ULL);
        tk = __shfl_sync(0xffffffff, tk, 0);
        for (int i = 0; i < 2; i++)
            if ((long long)(tk + i) < p.norder) P[np++] = (long long)(tk + i);
        if (np == 0) break;
        int last[2] = {-1, -1};
        for (int l = 0; l < p.L; l++) {
            const LayerP &L = p.layer[l];
            for (int i = 0; i < np; i++) {
                long long q = P[i];
                int blk[3];
                blk[2] = (int)(q % p.npb[2]); q /= p.npb[2];
                blk[1] = (int)(q % p.npb[1]); q /= p.npb[1];
                blk[0] = (int)(q % p.npb[0]);
                int lo[3], hi[3];
                region_of(p.layer, p.L, p.PB, blk, l, lo, hi);
                const int nsub = region_subtiles(L, lo, hi);
                const int wait = last[i];
                for (int k = 0; k < nsub; k++) {
                    const int kk = k / L.nnc, nc = k % L.nnc;
                    emit(l, ((((P[i] << 16) | kk) << 8 | nc) << 1) | i, wait);
                    last[i] = (int)qseq - 1;
                }
                computed += nsub;
            }
        }
    }
    emit(-1, 0, -1);
    (void)computed;
}

// Memoized scheduler (§3.2.2, Fig 2d), one warp.  Tickets are drawn along the host-built order
// (gen_task_order); a ticket's task is claimed with CAS 0 -> 1, its not-started dependencies are claimed
// recursively (the walk back of Fig 2d), and the bundle is handed to the loaders producers-first (layer order).
// A task is handed over only when it is READY: every dependency is published (state 2) or was handed over by this
// CTA earlier (state 3, ours; it completes ahead of the dependent in this CTA's in-order pipeline).  A claimed task
// whose dependency is still in progress on another CTA is not waited for: it goes to a pending list and is
// revisited later ("moves on ... and revisits this brick later", L523-525), so one slow tile never blocks the
// CTA's pipeline.  Progress: the lowest-layer pending task of all CTAs only depends on handed-over tasks.
// Tag word: (epoch << 10) | (owner CTA << 2) | state, state 0 free, 1 claimed, 3 claimed + handed over, 2 done.
__device__ void scheduler(const Params &p, Shared &sh) {
    const int lane = threadIdx.x % 32;
    const unsigned EP = run_epoch(p.counters) << 10;
    const int MINE1 = (int)(EP | (blockIdx.x << 2) | 1), MINE3 = (int)(EP | (blockIdx.x << 2) | 3);
    const bool unmerged = p.only_layer >= 0;
    unsigned long long oks = 0, defers = 0;
    uint32_t qseq = 0;
    auto emit = [&](int l, long long t) {
        const int slot = qseq % kQ;
        if (qseq >= (uint32_t)kQ) ptx::mbar_wait(&sh.q_empty[slot], ((qseq / kQ) - 1) & 1);
        if (lane == 0) {
            if (l >= 0 && !unmerged) atomicExch(status_word(p, l, t), MINE3);   // handed over (before any publish)
            sh.q_l[slot] = l;
            sh.q_t[slot] = t;
            sh.q_w[slot] = -1;
            mbar_arrive(&sh.q_full[slot]);
        }
        __syncwarp();
        qseq++;
    };
    if (unmerged) {
        for (;;) {
            unsigned long long tk = 0;
            if (lane == 0) tk = atomicAdd(&p.counters[4], 1ULL);
            tk = __shfl_sync(0xffffffff, tk, 0);
            if ((long long)tk >= p.norder) break;
            emit(p.only_layer, (long long)tk);
        }
        emit(-1, 0);
        return;
    }
    // every dependency published, or handed over by this CTA
    auto ready = [&](int l, long long t) {
        const Deps D = deps_of(p.layer, l, t);
        const int nd = D.ns + D.nr;
        bool ok = true;
        for (int i0 = 0; i0 < nd; i0 += 32) {
            const int i = i0 + lane;
            bool mine = true;
            if (i < nd) {
                int dl;
                const long long dt = dep_at(p.layer, D, i, dl);
                const int v = ld_acquire(status_word(p, dl, dt));
                mine = tag_state(v, EP) == 2 || v == MINE3;
            }
            ok = __all_sync(0xffffffff, mine) && ok;
        }
        return ok;
    };
    int np = 0;                  // pending (claimed, not handed over) tasks: sh.pend_l / sh.pend_t [0, np)
    bool tickets = true;
    unsigned sleep_ns = 32;
    for (;;) {
        // revisit the pending tasks (in claim order)
        if (np > 0) {
            int w = 0;
            for (int i = 0; i < np; i++) {
                const int l = sh.pend_l[i];
                const long long t = sh.pend_t[i];
                __syncwarp();
                if (ready(l, t)) {
                    emit(l, t);
                } else {
                    if (lane == 0) {
                        sh.pend_l[w] = l;
                        sh.pend_t[w] = t;
                    }
                    w++;
                }
                __syncwarp();
            }
            np = w;
        }
        if (!tickets || np >= kPendDraw) {
            if (!tickets && np == 0) break;
            __nanosleep(sleep_ns);            // everything pending waits on other CTAs: back off
            sleep_ns = min(sleep_ns * 2, 1024u);
            continue;
        }
        sleep_ns = 32;
        unsigned long long tk = 0;
        if (lane == 0) tk = atomicAdd(&p.counters[4], 1ULL);
        tk = __shfl_sync(0xffffffff, tk, 0);
        if ((long long)tk >= p.norder) {
            tickets = false;
            continue;
        }
        const int e = p.order[tk];
        const int l0 = e >> kTaskBits;
        const long long t0 = e & ((1 << kTaskBits) - 1);
        int ok = 0;
        if (lane == 0) {
            int *sw = status_word(p, l0, t0);
            const int cur = ld_acquire(sw);
            ok = tag_state(cur, EP) == 0 && atomicCAS(sw, cur, MINE1) == cur;
        }
        ok = __shfl_sync(0xffffffff, ok, 0);
        if (!ok) continue;   // already claimed (by a dependent's walk back)
        oks++;
        __syncwarp();   // every lane is done reading the previous bundle's stack (racecheck)
        if (lane == 0) {
            sh.stk_l[0] = l0;
            sh.stk_t[0] = t0;
        }
        int sp = 1;
        // walk back (Fig 2d): claim the not-started dependencies (input and residual producers), transitively
        for (int s = 0; s < sp; s++) {
            __syncwarp();
            const int sl = sh.stk_l[s];
            const long long st = sh.stk_t[s];
            const Deps D = deps_of(p.layer, sl, st);
            const int nd = D.ns + D.nr;
            for (int i0 = 0; i0 < nd; i0 += 32) {
                const int i = i0 + lane;
                int claimed = 0, dl = 0;
                long long dt = 0;
                if (i < nd && sp < kStack - 32) {
                    dt = dep_at(p.layer, D, i, dl);
                    int *dw = status_word(p, dl, dt);
                    const int cur = ld_acquire(dw);
                    if (tag_state(cur, EP) == 0 && atomicCAS(dw, cur, MINE1) == cur) claimed = 1;
                }
                const unsigned cm = __ballot_sync(0xffffffff, claimed);
                oks += __popc(cm);
                if (claimed) {
                    const int pos = sp + __popc(cm & ((1u << lane) - 1));
                    sh.stk_l[pos] = dl;
                    sh.stk_t[pos] = dt;
                }
                sp += __popc(cm);
            }
        }
        __syncwarp();
        // hand the bundle over producers first (layers are listed topologically), deferring what is not ready
        for (int l = 0; l < p.L; l++) {
            for (int s = 0; s < sp; s++) {
                if (sh.stk_l[s] != l) continue;   // (warp-uniform: every lane reads the same entry)
                const long long t = sh.stk_t[s];
                __syncwarp();
                if (!p.defer || ready(l, t)) {
                    emit(l, t);
                } else {
                    defers++;
                    if (lane == 0) {
                        sh.pend_l[np] = l;
                        sh.pend_t[np] = t;
                    }
                    np++;
                }
                __syncwarp();
            }
        }
    }
    emit(-1, 0);
    if (lane == 0) {
        if (oks) atomicAdd(&p.counters[1], oks);
        if (defers) atomicAdd(&p.counters[2], defers);
    }
}

// ---------------------------------------------------------------------------------------------- loader
// One K-block of the input tile of a tile into stage `buf` (128 threads).  Positions outside the feature
// map (and, in padded mode, outside the source region) are zero-filled.
__device__ __forceinline__ void load_stage(const Params &p, const LayerP &L, const Tile &T, int kb, uint8_t *buf,
                                           int tid, uint64_t *bar) {
    // Row-by-row: loader warp w takes input rows (plane a, row yy) w, w + 4, ...; per row the brick-row
    // and scratch-row address arithmetic is done once, and the lanes walk (column, 16-B chunk) pairs with
    // shifts only (power-of-two brick extents, stride 1 or 2, chunk counts a power of two).
    const TView &v = L.src;
    const __nv_bfloat16 *base = reinterpret_cast<const __nv_bfloat16 *>(v.ptr);
    const __nv_bfloat16 *sbase = nullptr;
    int sp1 = 0, sp2 = 0;
    if (T.src_scr) {
        const LayerP &S = p.layer[&L - p.layer - 1];
        sbase = reinterpret_cast<const __nv_bfloat16 *>(scr_slot(p, T.slot) + S.scr_off);
        sp1 = S.pR[1];
        sp2 = S.pR[2];
    }
    const int lane = tid & 31, w = tid >> 5;
    const int lkc = L.lkc, kc = 1 << lkc;
    const int nrow = (L.ke[0] + L.Td - 1) * L.in_rows;   // input planes x rows (Td output planes per task)
    const int z0 = T.d * L.s[0] - L.pd[0];
    const int y0 = T.y0 * L.s[1] - L.pd[1];
    const int x0 = T.x0 * L.s[2] - L.pd[2];
    const uint32_t plane_bytes = (uint32_t)L.rowsA * 16;
    const int ls2 = L.s[2] - 1;                   // log2 of the column stride (1 or 2)
    const int lBd = L.lB[0], lBh = L.lB[1], lBw = L.lB[2];
    const int nchunk = L.in_cols << lkc;
    if (L.tma == 2 && !T.src_scr) {
        // 1x1 stride-2 SW128 layer: only polyphase block (0, 0) is read by the MMAs.  Output row i reads input
        // row 2 * (y0 + i); one TMA box per row picks every other pixel (element stride 2 along x in brick)
        // and lands the Tw pixels contiguously at block row i.
        const int l = (int)(&L - p.layer);
        for (int i = w; i < L.Tb; i += kLW) {
            const int y = y0 + 2 * i;
            uint8_t *dst = buf + (size_t)(i * L.Wp) * 128;
            if (y >= 0 && y < L.in_ext[1]) {
                if (lane == 0) {
                    ptx::mbar_expect_tx(bar, (uint32_t)L.Tw * 128);
                    const int by = y >> lBh;
                    ptx::tma_load_5d(dst, &p.tm_row[l], kb * 64, 0, x0 >> lBw, y - (by << lBh),
                                     T.n * v.nb[2] + by, bar);
                }
            } else {
                for (int q = lane; q < L.Tw * 8; q += 32)
                    *reinterpret_cast<uint4 *>(dst + (size_t)(q >> 3) * 128 + ((q & 7) << 4)) = make_uint4(0, 0, 0, 0);
            }
        }
        ptx::fence_proxy_async_smem();
        return;
    }
    if (L.tma == 3 && !T.src_scr) {
        // 3x3 stride-2 SW128 layer (padding 1): polyphase block (yr, xr) holds input pixels (2 yq + yr, 2 xq + xr) of the
        // window starting at (y0, x0) = (2 Y - 1, 2 X - 1).  Per input row, two TMA boxes with element stride 2 along x
        // fetch the Tw interior even columns 2X, 2X + 2, ... into block (yr, 1) at xq = 0..Tw-1 and the Tw odd columns
        // 2X + 1, ... into block (yr, 0) at xq = 1..Tw; the two halo pixels 2X - 1 (block (yr, 0), xq 0) and 2X + 2Tw
        // (block (yr, 1), xq Tw) come by cp.async; rows outside the image are zero-filled.
        const int l = (int)(&L - p.layer);
        const int X = T.x0 * 2;   // first interior input column: brick aligned (Tw % Bw == 0)
        for (int yy = w; yy < L.in_rows; yy += kLW) {
            const int y = y0 + yy;
            const int rowpx0 = (yy & 1) * 2 * L.blk_px + (yy >> 1) * L.Wp, rowpx1 = rowpx0 + L.blk_px;
            const bool rok = y >= 0 && y < L.in_ext[1];
            const int by = y >> lBh, yin = y - (by << lBh);
            if (rok) {
                if (lane == 0) {
                    ptx::mbar_expect_tx(bar, 2u * (uint32_t)L.Tw * 128u);
                    ptx::tma_load_5d(buf + (size_t)rowpx1 * 128, &p.tm_row[l], kb * 64, 0, X >> lBw, yin,
                                     T.n * v.nb[2] + by, bar);
                    ptx::tma_load_5d(buf + (size_t)(rowpx0 + 1) * 128, &p.tm_row[l], kb * 64, 1, X >> lBw, yin,
                                     T.n * v.nb[2] + by, bar);
                }
            } else {
                for (int q = lane; q < 2 * L.Tw * 8; q += 32) {
                    const int px = q < L.Tw * 8 ? rowpx1 + (q >> 3) : rowpx0 + 1 + ((q - L.Tw * 8) >> 3);
                    *reinterpret_cast<uint4 *>(buf + (size_t)px * 128 + (((q & 7) ^ (px & 7)) << 4)) = make_uint4(0, 0, 0, 0);
                }
            }
            if (lane < 16) {   // halo pixels: 8 16-B chunks each
                const int side = lane >> 3, ch = lane & 7;
                const int x = side ? X + 2 * L.Tw : X - 1;
                const int px = side ? rowpx1 + L.Tw : rowpx0;
                const bool ok = rok && x >= 0 && x < L.in_ext[2];
                const void *g = base;
                if (ok) {
                    const int bx = x >> lBw;
                    g = base + ((((long long)T.n * v.nb[1]) * v.nb[2] + by) * v.nb[3] + bx) * v.brick_elems +
                        (long long)((yin << lBw) + (x - (bx << lBw))) * v.Cp + kb * 64 + ch * 8;
                }
                ptx::cp_async16(buf + (size_t)px * 128 + ((ch ^ (px & 7)) << 4), g, ok ? 16u : 0u);
            }
        }
        ptx::fence_proxy_async_smem();   // zero-filled rows (generic stores) -> tcgen05 operand reads
        return;
    }
    if (L.tma == 4 && !T.src_scr) {
        // 1x1 stride-1 layer whose tiles start on a brick row (Tb % Bh == 0, no halo: Wp == Tw): the Bh rows of a brick
        // row of bricks land as Bh consecutive tile rows of Tw pixels, one TMA box each; rows past the bricked grid are
        // zero-filled by TMA's out-of-bounds fill
        const int l = (int)(&L - p.layer);
        const int Bh = 1 << lBh;
        for (int b = w; b < (L.Tb >> lBh); b += kLW) {
            if (lane == 0) {
                ptx::mbar_expect_tx(bar, (uint32_t)(Bh * L.Tw) * 128u);
                ptx::tma_load_5d(buf + (size_t)(b * Bh * L.Wp) * 128, &p.tm_row[l], kb * 64, 0, T.x0 >> lBw, 0,
                                 T.n * v.nb[2] + (y0 >> lBh) + b, bar);
            }
        }
        return;
    }
    if (L.tma && !T.src_scr) {
        // stride-1 swizzled rows (SW128: 64-channel K-block rows of 128 B; SW64: 32-channel rows of 64 B): the
        // Tw in-tile columns of an in-image row by one TMA box (completion on `bar` by transaction count), halo
        // columns by cp.async into the same swizzled layout, rows outside the image zero-filled
        const int l = (int)(&L - p.layer);
        const int pdw = L.pd[2];
        const int nh = L.in_cols - L.Tw;          // halo columns (k - 1)
        const bool sw64 = L.amode == AM_SW64;
        const int rb = sw64 ? 64 : 128, lrb = sw64 ? 6 : 7, nchr = sw64 ? 4 : 8;   // row bytes, log2, chunks / row
        // SW64 (32-channel, typically 3-D: many short rows): one input row per loader THREAD, so the per-row
        // address arithmetic of the ~50 rows runs in parallel; SW128 (64-channel K-blocks, 2-D: few rows with
        // 16 halo chunks each): one row per WARP with the lanes on the halo chunks.  Measured on B200: cfg5
        // 2.45 -> 2.04 ms with per-thread rows, while per-thread rows cost cfg3 / cfg4 1.5-3.5 %.
        const int rstep = sw64 ? kLoadT : kLW, rbeg = sw64 ? tid : w;
        const int hstep = sw64 ? 1 : 32, hbeg = sw64 ? 0 : lane;
        for (int r2 = rbeg; r2 < nrow; r2 += rstep) {
            const int a = r2 / L.in_rows, yy = r2 - a * L.in_rows;
            const int z = z0 + a, y = y0 + yy;
            const bool rok = z >= 0 && z < L.in_ext[0] && y >= 0 && y < L.in_ext[1];
            const int rowpx = a * L.plane_px + yy * L.Wp + L.pxo;
            const int bz = z >> lBd, by = y >> lBh;
            if (rok) {
                if (hbeg == 0) {
                    ptx::mbar_expect_tx(bar, (uint32_t)(L.Tw * rb));
                    ptx::tma_load_5d(buf + ((size_t)(rowpx + pdw) << lrb), &p.tm_row[l], kb * 64, 0, T.x0 >> lBw,
                                     ((z - (bz << lBd)) << lBh) + (y - (by << lBh)),
                                     (T.n * v.nb[1] + bz) * v.nb[2] + by, bar);
                }
            } else {
                for (int q = hbeg; q < L.Tw * nchr; q += hstep)
                    *reinterpret_cast<uint4 *>(buf + ((size_t)(rowpx + pdw) << lrb) + ((size_t)q << 4)) =
                        make_uint4(0, 0, 0, 0);
            }
            const long long rowlog = (((long long)T.n * v.nb[1] + bz) * v.nb[2] + by) * v.nb[3];
            const int rowin = ((z - (bz << lBd)) << lBh) + (y - (by << lBh));
            for (int q = hbeg; q < nh * nchr; q += hstep) {
                const int hc = q / nchr, ch = q - hc * nchr;
                const int xx = hc < pdw ? hc : L.Tw + hc;
                const int x = x0 + xx;
                const bool ok = rok && x >= 0 && x < L.in_ext[2];
                const int px = rowpx + xx;
                const int bx = x >> lBw;
                const void *g = base;
                if (ok)
                    g = base + (rowlog + bx) * v.brick_elems + (long long)((rowin << lBw) + (x - (bx << lBw))) * v.Cp +
                        kb * 64 + ch * 8;
                const uint32_t off = sw64 ? (uint32_t)px * 64 + ((ch ^ ((px >> 1) & 3)) << 4)
                                          : (uint32_t)px * 128 + ((ch ^ (px & 7)) << 4);
                ptx::cp_async16(buf + off, g, ok ? 16u : 0u);
            }
        }
        ptx::fence_proxy_async_smem();   // zero-filled rows (generic stores) -> tcgen05 operand reads
        return;
    }
    for (int r2 = w; r2 < nrow; r2 += kLW) {
        const int a = r2 / L.in_rows, yy = r2 - a * L.in_rows;
        const int z = z0 + a, y = y0 + yy;
        bool rok = z >= 0 && z < L.in_ext[0] && y >= 0 && y < L.in_ext[1];
        if (T.src_scr) rok = rok && z >= T.slo[0] && z < T.shi[0] && y >= T.slo[1] && y < T.shi[1];
        const int yq = L.s[1] == 2 ? (yy >> 1) : yy, yr = L.s[1] == 2 ? (yy & 1) : 0;
        const int rowpx = a * L.plane_px + yr * L.s[2] * L.blk_px + yq * L.Wp;
        long long rowlog = 0, srow = 0;
        int rowin = 0;
        if (rok) {
            if (T.src_scr) {
                srow = ((long long)(z - T.slo[0]) * sp1 + (y - T.slo[1])) * sp2;
            } else {
                const int bd = z >> lBd, by = y >> lBh;
                rowlog = (((long long)T.n * v.nb[1] + bd) * v.nb[2] + by) * v.nb[3];
                rowin = (((z - (bd << lBd)) << lBh) + (y - (by << lBh))) << lBw;
            }
        }
        for (int q = lane; q < nchunk; q += 32) {
            const int xx = q >> lkc, ch = q & (kc - 1);
            const int x = x0 + xx;
            bool ok = rok && x >= 0 && x < L.in_ext[2];
            if (T.src_scr) ok = ok && x >= T.slo[2] && x < T.shi[2];
            const int px = rowpx + (xx & ls2) * L.blk_px + (xx >> ls2);
            uint32_t off;
            if (L.amode == AM_SW128) off = (uint32_t)px * 128 + ((ch ^ (px & 7)) << 4);
            else if (L.amode == AM_SW64) {
                const int pq = px + L.pxo;
                off = (uint32_t)pq * 64 + ((ch ^ ((pq >> 1) & 3)) << 4);
            }
            else off = (uint32_t)ch * plane_bytes + (uint32_t)px * 16;
            const void *g = base;
            if (ok) {
                if (T.src_scr) {
                    g = sbase + ((srow + (x - T.slo[2])) * L.cin + kb * 64 + ch * 8);
                } else {
                    const int bx = x >> lBw;
                    const long long logical = rowlog + bx;
                    const long long phys = v.bmap ? (long long)v.bmap[logical] : logical;
                    g = base + phys * v.brick_elems + (long long)(rowin + x - (bx << lBw)) * v.Cp + kb * 64 + ch * 8;
                }
            }
            ptx::cp_async16(buf + off, g, ok ? 16u : 0u);
        }
    }
}

// 256-bit global accesses (sm_100): one full 32-B sector per lane
__device__ __forceinline__ void ld_cg_v8(const uint4 *p, uint32_t (&r)[8]) {
    asm volatile("ld.global.cg.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "l"(p));
}
__device__ __forceinline__ void st_v8(uint4 *p, const uint32_t (&w)[8]) {
    asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(w[0]), "r"(w[1]), "r"(w[2]),
                 "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7])
                 : "memory");
}
// the same with an L2 eviction-priority policy (createpolicy): locality-aware memoization keeps the memo buffers
// that later layers of the subgraph read resident and streams the subgraph's outputs
__device__ __forceinline__ void st_v8_pol(uint4 *p, const uint32_t (&w)[8], uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8}, %9;" ::"l"(p), "r"(w[0]), "r"(w[1]),
                 "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7]), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ uint32_t pack2(float a, float b) {
    __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<uint32_t *>(&v);
}

// One stacked k-step (not the first: every MMA accumulates), input planes and M tiles unrolled: per input plane i the
// D column, B row offset and instruction descriptor are loop-invariant (precomputed by the caller), so the issue chain
// is two 64-bit adds per MMA.
template <int TD, int NTL>
__device__ __forceinline__ void issue_stacked_q(uint64_t adq, uint64_t bd, uint32_t d_base, const uint32_t *col,
                                                const uint64_t *bo, const uint32_t *idn, uint64_t pstep, uint64_t astep,
                                                uint32_t tstep) {
#pragma unroll
    for (int i = 0; i < TD + 2; i++)
#pragma unroll
        for (int tl = 0; tl < NTL; tl++)
            ptx::mma_bf16_elect_nc(d_base + tl * tstep + col[i], adq + i * pstep + tl * astep, bd + bo[i], idn[i], 1u);
}

// ---------------------------------------------------------------------------------------------- kernel
// Unstacked k-steps [q0, q1) of a swizzled-A layer with every MMA accumulating (the caller peels a task's first
// k-step), M tiles unrolled: one table load and one add per k-step, then NTL issues (measured: VGG-16 -3 %).
template <int NTL>
__device__ __forceinline__ void issue_ksteps(const uint32_t *ksl, int q0, int q1, uint64_t a_d0, uint64_t bd, uint32_t ks_u,
                                             uint32_t d_base, uint32_t dstep, uint64_t astep, uint32_t idesc) {
#pragma unroll 4
    for (int q = q0; q < q1; q++, bd += ks_u) {
        const uint64_t ad = a_d0 + (ksl[q] & 0xFFFFu);
#pragma unroll
        for (int tl = 0; tl < NTL; tl++) ptx::mma_bf16_elect_nc(d_base + tl * dstep, ad + tl * astep, bd, idesc, 1u);
    }
}

// STK: the subgraph has depth-stacked layers.  Two instantiations, so the stacked issue path is absent from the kernel
// that 2-D subgraphs run (present, it cost 2-D layers ~15 % through the MMA warp's register allocation; B200 A/B).
template <bool STK, int EPIW>
__global__ void __launch_bounds__(32 * (kEpi0 + EPIW), 1) gen_kernel(const __grid_constant__ Params p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ Shared sh;
    const int warp = __shfl_sync(0xffffffff, (int)threadIdx.x / 32, 0), lane = threadIdx.x % 32;
    uint8_t *in_ring = smem;
    uint8_t *w_ring = smem + (size_t)p.nin * p.in_stride;
    if (ptx::smem_u32(smem) & 1023) __trap();   // 128-B swizzle atoms need 1024-B alignment

    // k-step descriptor-offset tables
    for (int i = threadIdx.x; i < p.L * kMaxKs; i += (32 * (kEpi0 + EPIW))) {
        const int l = i / kMaxKs, q = i % kMaxKs;
        const LayerP &L = p.layer[l];
        if (q >= (L.stk ? L.nks / L.k[0] : L.nks)) continue;
        int tap, kk = 0, t1 = -1;
        // stacked 3-D layers: the table holds the k0 = 1 view (r, s, kk); the depth tap picks the input plane at issue
        const int k0t = L.stk ? 1 : L.k[0];
        if (L.amode == AM_SW128) kstep_tap(q, k0t, L.k[1], L.k[2], 4, tap, kk);
        else if (L.amode == AM_SW64) kstep_tap(q, k0t, L.k[1], L.k[2], 2, tap, kk);
        else if (L.amode == AM_PLANES) kstep_tap(q, k0t, L.k[1], L.k[2], (L.cin + 15) / 16, tap, kk);
        else {   // pair taps (a, r, 2u) and (a, r, 2u+1)
            const int np = (L.k[2] + 1) / 2;
            const int u = q % np, ar = q / np;
            tap = ar * L.k[2] + 2 * u;
            t1 = 2 * u + 1 < L.k[2] ? tap + 1 : -1;
        }
        auto tap_px = [&](int tp) {
            // tap (a, r, s) reads input offset (a*dl0, r*dl1, s*dl2) of the output position: its polyphase block and
            // row / column inside the block
            const int s = (tp % L.k[2]) * L.dl[2], r = ((tp / L.k[2]) % L.k[1]) * L.dl[1],
                      a = (tp / (L.k[2] * L.k[1])) * L.dl[0];
            return a * L.plane_px + ((r % L.s[1]) * L.s[2] + (s % L.s[2])) * L.blk_px + (r / L.s[1]) * L.Wp + s / L.s[2];
        };
        uint32_t aoff, lbo;
        if (L.amode == AM_SW128) { aoff = (uint32_t)tap_px(tap) * 8 + kk * 2; lbo = 1; }
        else if (L.amode == AM_SW64) { aoff = (uint32_t)(tap_px(tap) + L.pxo) * 4 + kk * 2; lbo = 1; }
        else if (L.amode == AM_PLANES) { aoff = (uint32_t)tap_px(tap) + 2u * kk * L.rowsA; lbo = L.rowsA; }
        else { aoff = tap_px(tap); lbo = t1 >= 0 ? (uint32_t)(tap_px(t1) - tap_px(tap)) : 0u; }
        sh.ks[l][q] = (aoff & 0xFFFF) | (lbo << 16);
    }
    if (p.bias_off >= 0) {   // the biases are weights (not the previous kernel's output): staged before the PDL wait
        float *bt = reinterpret_cast<float *>(smem + p.bias_off);
        for (int l = 0; l < p.L; l++)
            for (int c = threadIdx.x; c < p.layer[l].cout; c += 32 * (kEpi0 + EPIW)) bt[p.layer[l].bofs + c] = p.layer[l].bias[c];
    }
    if (threadIdx.x == 0) {
        for (int i = 0; i < kQ; i++) {
            ptx::mbar_init(&sh.q_full[i], 1);
            ptx::mbar_init(&sh.q_empty[i], 2);          // loader + weight producer
        }
        for (int i = 0; i < kMaxIn; i++) {
            ptx::mbar_init(&sh.in_full[i], kLoadT);      // every loader thread after its copies landed
            ptx::mbar_init(&sh.in_empty[i], 1);
        }
        for (int i = 0; i < kMaxW; i++) {
            ptx::mbar_init(&sh.wfull[i], 1);
            ptx::mbar_init(&sh.wempty[i], 1);
        }
        for (int i = 0; i < 2; i++) {
            ptx::mbar_init(&sh.acc_full[i], 1);
            ptx::mbar_init(&sh.acc_empty[i], EPIW);
        }
        for (int i = 0; i < kRing; i++) ptx::mbar_init(&sh.desc_full[i], 1);
        sh.done_seq = 0;
        ptx::fence_barrier_init();
    }
    if (warp == kMma) {
        ptx::tmem_alloc(&sh.tmem_base, p.tmem_cols);
        ptx::tmem_relinquish();
    }
    ptx::fence_proxy_async_smem();
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
    pdl_launch_dependents();
    // loaders / epilogue read the previous kernel's output; the scheduler rewrites memo tags that a previous
    // run of this subgraph may still be waiting on
    const bool waits = (warp >= kLoad0 && warp < kLoad0 + kLW) || warp >= kEpi0 || warp == kSched;
    if (waits) pdl_wait();

    const unsigned EP = waits ? run_epoch(p.counters) << 10 : 0u;   // tag word: epoch << 10 | owner << 2 | state
    if (warp == kSched) {
        if (p.padded) scheduler_padded(p, sh);
        else scheduler(p, sh);
    } else if (warp < kLoad0 + kLW) {
        // ------------------------------------------------------------------ loaders
        const int tid = threadIdx.x - 32 * kLoad0;
        uint32_t gin = 0;
        unsigned long long wq = 0, wdep = 0, wbuf = 0, wiss = 0, wbar = 0;
        const unsigned long long t_start = clock64();
        for (uint32_t seq = 0;; seq++) {
            const int slot = seq % kQ;
            pwait(p, &sh.q_full[slot], (seq / kQ) & 1, wq);
            const int l = sh.q_l[slot];
            const long long t = sh.q_t[slot];
            const int wait = sh.q_w[slot];
            if (l > 0 && p.padded && wait >= 0 && warp == kLoad0) {
                // padded: the source region is written by this CTA's epilogue of sub-task `wait`
                if (lane == 0) {
                    // atomic read of the CTA-local flag (release/acquire through fences around CTA-scope atomics)
                    while (atomicOr_block(&sh.done_seq, 0) <= wait) __nanosleep(64);
                    __threadfence();
                }
                __syncwarp();
            } else if (l >= 0 && !p.padded && p.only_layer < 0 && warp == kLoad0) {
                // wait for the dependency tiles of the input and residual producers (state 2 of this epoch)
                const Deps D = deps_of(p.layer, l, t);
                const int nd = D.ns + D.nr;
                unsigned long long spins = 0;
                const unsigned long long td0 = clock64();
                for (int i = lane; i < nd; i += 32) {
                    int dl;
                    const long long dt = dep_at(p.layer, D, i, dl);
                    const int *dw = status_word(p, dl, dt);
                    while (ld_acquire(dw) != (int)(EP | 2)) {
                        spins++;
                        __nanosleep(32);
                    }
                }
                __syncwarp();
                wdep += clock64() - td0;
                for (int o = 16; o; o >>= 1) spins += __shfl_xor_sync(0xffffffff, spins, o);
                if (lane == 0 && spins) atomicAdd(&p.counters[3], spins);
            }
            PT(const unsigned long long tlb = p.prof ? clock64() : 0;)
            asm volatile("bar.sync 1, %0;" ::"n"(kLoadT) : "memory");
            PT(if (p.prof) wbar += clock64() - tlb;)
            // acquired data (generic-proxy stores of other CTAs) is read by TMA (async proxy); a source written by an earlier
            // grid needs no fence, and the global-memory proxy fence is the one needed (the full fence: ~1 us per task)
            if (l >= 0 && p.layer[l].tma && p.layer[l].srcl >= 0 && !p.padded) asm volatile("fence.proxy.async.global;" ::: "memory");
            if (tid == 0) {
                sh.desc_l[seq % kRing] = l;
                sh.desc_t[seq % kRing] = t;
                mbar_arrive(&sh.desc_full[seq % kRing]);
                mbar_arrive(&sh.q_empty[slot]);
            }
            if (l < 0) break;
            const LayerP &L = p.layer[l];
            const Tile T = make_tile(p, l, t);
            for (int kb = 0; kb < L.nkb; kb++, gin++) {
                const int s = gin % p.nin;
                if (gin >= (uint32_t)p.nin) pwait(p, &sh.in_empty[s], ((gin / p.nin) - 1) & 1, wbuf);
                PT(const unsigned long long tl0 = p.prof ? clock64() : 0;)
                if (!DBG(p, 2)) load_stage(p, L, T, kb, in_ring + (size_t)s * p.in_stride, tid, &sh.in_full[s]);
                PT(if (p.prof) wiss += clock64() - tl0;)
                // completion tracked by the barrier (the loader moves on to the next stage / task at once)
                ptx::cp_async_arrive_noinc(&sh.in_full[s]);
            }
        }
        if (p.prof && tid == 0) {
            unsigned long long *r = p.prof + (size_t)blockIdx.x * 32;
            r[0] = wq; r[1] = wdep; r[2] = wbuf; r[3] = clock64() - t_start; r[20] = wiss; r[21] = wbar;
        }
    } else if (warp == kWProd) {
        // ------------------------------------------------------------------ weight producer
        uint32_t gw = 0;
        unsigned long long ww = 0;
        const unsigned long long t_start = clock64();
        for (uint32_t seq = 0;; seq++) {
            const int slot = seq % kQ;
            ptx::mbar_wait(&sh.q_full[slot], (seq / kQ) & 1);
            // lane 0 reads the queue entry and releases the slot; the warp gets it by shuffle
            int l = 0;
            long long t = 0;
            if (lane == 0) {
                l = sh.q_l[slot];
                t = sh.q_t[slot];
                mbar_arrive(&sh.q_empty[slot]);
            }
            l = __shfl_sync(0xffffffff, l, 0);
            t = __shfl_sync(0xffffffff, t, 0);
            if (l < 0) break;
            const LayerP &L = p.layer[l];
            const int nc = p.padded ? (int)((t >> 1) & 0xFF) : (int)((unsigned)t % (unsigned)L.nnc);
            const size_t ks_bytes = (size_t)2 * (L.stk ? 3 : 1) * L.Nc * 16;   // stacked: three depth taps per k-step
            const int nqs = L.stk ? L.nks / 3 : L.nks;
            const uint8_t *wl = reinterpret_cast<const uint8_t *>(L.w) + (size_t)nc * L.nkb * nqs * ks_bytes;
            for (int kb = 0; kb < L.nkb; kb++) {
                for (int j = 0; j < L.nws; j++, gw++) {
                    const int st = gw % p.nw;
                    const int q0 = j * L.kpw, nq = min(L.kpw, nqs - q0);
                    const uint32_t bytes = (uint32_t)(nq * ks_bytes);
                    if (gw >= (uint32_t)p.nw) pwait(p, &sh.wempty[st], ((gw / p.nw) - 1) & 1, ww);
                    if (ptx::elect_one()) {
                        ptx::mbar_arrive_expect_tx(&sh.wfull[st], bytes);
                        ptx::bulk_g2s(w_ring + (size_t)st * p.w_stride, wl + ((size_t)kb * nqs + q0) * ks_bytes, bytes,
                                      &sh.wfull[st]);
                    }
                    __syncwarp();
                }
            }
        }
        if (p.prof && lane == 0) {
            unsigned long long *r = p.prof + (size_t)blockIdx.x * 32;
            r[4] = ww; r[5] = clock64() - t_start;
        }
    } else if (warp == kMma) {
        // ------------------------------------------------------------------ MMA issuer
        const uint32_t tmem_base = __shfl_sync(0xffffffff, sh.tmem_base, 0);
        uint32_t gin = 0, gw = 0;
        unsigned long long wdesc = 0, wacc = 0, win = 0, wwt = 0, wfence = 0;
        const unsigned long long t_start = clock64();
        for (uint32_t seq = 0;; seq++) {
            pwait(p, &sh.desc_full[seq % kRing], (seq / kRing) & 1, wdesc);
            const int l = sh.desc_l[seq % kRing];
            if (l < 0) break;
            const LayerP &L = p.layer[l];
            const int a = seq % p.nacc;
            if (seq >= (uint32_t)p.nacc) pwait(p, &sh.acc_empty[a], ((seq / p.nacc) - 1) & 1, wacc);
            ptx::tc_fence_after();
            const uint32_t d_base = tmem_base + a * p.acc_stride;
            const uint32_t nbr = (uint32_t)(L.stk ? 3 : 1) * L.Nc;   // B rows per k-step (stacked: three depth taps)
            const uint32_t lbo_b = nbr * 16;
            const uint32_t ks_u = nbr * 2;   // 16-B units per k-step of B
            // issue constants hoisted out of the k-step loop; descriptors advance by 64-bit adds (start-address fields
            // stay below 2^14 16-B units: shared memory < 256 KB)
            const int ntl = L.ntl;
            const uint32_t idesc = L.idesc, dstep = (uint32_t)L.Nc;
            const uint64_t astep = 128ull * (uint64_t)L.row_u;
            const bool noswz = L.amode != AM_SW128 && L.amode != AM_SW64;
            const uint64_t ad_t = L.amode == AM_SW128 ? ptx::umma_desc_sw128(0, 1024)
                                  : L.amode == AM_SW64 ? ptx::umma_desc_sw64(0, 512)
                                                       : ptx::umma_desc_noswz(0, 0, 128);
            const uint64_t bd_t = ptx::umma_desc_noswz(0, lbo_b, 128);
            const uint32_t *ksl = sh.ks[l];
            for (int kb = 0; kb < L.nkb; kb++, gin++) {
                const int s = gin % p.nin;
                pwait(p, &sh.in_full[s], (gin / p.nin) & 1, win);
                const unsigned long long tf0 = p.prof ? clock64() : 0;
                ptx::fence_proxy_async_smem();   // cp.async (generic proxy) data -> tcgen05 operand reads
                ptx::tc_fence_after();
                if (p.prof) wfence += clock64() - tf0;
                const uint32_t a_base = ptx::smem_u32(in_ring + (size_t)s * p.in_stride) >> 4;
                for (int j = 0; j < L.nws; j++, gw++) {
                    const int st = gw % p.nw;
                    pwait(p, &sh.wfull[st], (gw / p.nw) & 1, wwt);
                    ptx::tc_fence_after();
                    const uint32_t b_base = ptx::smem_u32(w_ring + (size_t)st * p.w_stride) >> 4;
                    const int q0 = j * L.kpw, q1 = DBG(p, 1) ? q0 + 1 : min(L.stk ? L.nks / 3 : L.nks, q0 + L.kpw);
                    const uint64_t a_d0 = ad_t + a_base;
                    uint64_t bd = bd_t + b_base;
                    if (STK && L.stk) {
                        // depth-stacked 3-D layer: per k-step (r, s, kk), input plane i feeds output planes o = i - a for the
                        // depth taps a in [alo, ahi]: ONE MMA with N = (ahi - alo + 1) Nc, B = those taps' weights side
                        // by side, D = the planes' accumulators, laid out at columns (Td - 1 - o) Nc so they are contiguous
                        // and ascending.  The first k-step gives each plane's first product (a = 0) its own MMA without
                        // accumulate.  Per output element the order is (r, s, kk) outer, a inner -- the unstacked order.
                        const int Td = L.Td, Nc = L.Nc;
                        const uint64_t pstep = (uint64_t)L.plane_px * (uint64_t)L.row_u;
                        const uint32_t tstep = (uint32_t)(Td * Nc);
                        auto issue_n = [&](uint64_t ad, uint64_t bdd, int o_hi, int na, uint32_t acc) {
                            const uint32_t col = (uint32_t)((Td - 1 - o_hi) * Nc);
                            const uint32_t idn = L.idesc_s[na - 1];
                            for (int tl = 0; tl < ntl; tl++)
                                ptx::mma_bf16_elect_nc(d_base + tl * tstep + col, ad + tl * astep, bdd, idn, acc);
                        };
                        // per input plane: D column, B row offset, descriptor (loop-invariant over the k-steps)
                        uint32_t colv[6], idnv[6];
                        uint64_t bov[6];
#pragma unroll
                        for (int i = 0; i < 6; i++) {
                            const int alo = max(0, i - Td + 1), ahi = min(2, i);
                            colv[i] = (uint32_t)((Td - 1 - (i - alo)) * Nc);
                            bov[i] = (uint64_t)(alo * Nc);
                            idnv[i] = L.idesc_s[max(0, min(2, ahi - alo))];
                        }
                        const bool fast = !noswz && (Td == 1 || Td == 2 || Td == 4) && (ntl == 1 || ntl == 2);
                        for (int q = q0; q < q1; q++, bd += ks_u) {
                            const uint32_t ev = ksl[q];
                            const uint64_t adq = noswz ? (ad_t | ((uint64_t)(ev >> 16) << 16)) + a_base + (ev & 0xFFFF)
                                                       : a_d0 + (ev & 0xFFFFu);
                            const bool first = (kb | q) == 0;
                            if (fast && !first) {
                                if (Td == 1 && ntl == 1) issue_stacked_q<1, 1>(adq, bd, d_base, colv, bov, idnv, pstep, astep, tstep);
                                else if (Td == 1) issue_stacked_q<1, 2>(adq, bd, d_base, colv, bov, idnv, pstep, astep, tstep);
                                else if (Td == 2 && ntl == 1) issue_stacked_q<2, 1>(adq, bd, d_base, colv, bov, idnv, pstep, astep, tstep);
                                else if (Td == 2) issue_stacked_q<2, 2>(adq, bd, d_base, colv, bov, idnv, pstep, astep, tstep);
                                else if (ntl == 1) issue_stacked_q<4, 1>(adq, bd, d_base, colv, bov, idnv, pstep, astep, tstep);
                                else issue_stacked_q<4, 2>(adq, bd, d_base, colv, bov, idnv, pstep, astep, tstep);
                                continue;
                            }
                            for (int i = 0; i < Td + 2; i++) {
                                const int alo = max(0, i - Td + 1), ahi = min(2, i);
                                const uint64_t ad = adq + i * pstep;
                                if (first && alo == 0) {
                                    issue_n(ad, bd, i, 1, 0u);
                                    if (ahi >= 1) issue_n(ad, bd + (uint64_t)Nc, i - 1, ahi, 1u);
                                } else {
                                    issue_n(ad, bd + (uint64_t)(alo * Nc), i - alo, ahi - alo + 1, 1u);
                                }
                            }
                        }
                        ptx::mma_commit_elect(&sh.wempty[st]);
                        continue;
                    }
                    auto issue = [&](uint64_t ad, uint32_t acc) {
                        ptx::mma_bf16_elect_nc(d_base, ad, bd, idesc, acc);
                        if (ntl > 1) ptx::mma_bf16_elect_nc(d_base + dstep, ad + astep, bd, idesc, acc);
                        if (ntl > 2) ptx::mma_bf16_elect_nc(d_base + 2 * dstep, ad + 2 * astep, bd, idesc, acc);
                        if (ntl > 3)
                            for (int tl = 3; tl < ntl; tl++)
                                ptx::mma_bf16_elect_nc(d_base + tl * dstep, ad + tl * astep, bd, idesc, acc);
                    };
                    if (noswz) {
                        for (int q = q0; q < q1; q++, bd += ks_u) {
                            const uint32_t ev = ksl[q];
                            issue((ad_t | ((uint64_t)(ev >> 16) << 16)) + a_base + (ev & 0xFFFF), (kb | q) != 0);
                        }
                    } else {
                        int qs = q0;
                        if ((kb | q0) == 0 && q0 < q1) {
                            issue(a_d0 + (ksl[q0] & 0xFFFFu), 0u);
                            qs++;
                            bd += ks_u;
                        }
                        if (ntl == 1) issue_ksteps<1>(ksl, qs, q1, a_d0, bd, ks_u, d_base, dstep, astep, idesc);
                        else if (ntl == 2) issue_ksteps<2>(ksl, qs, q1, a_d0, bd, ks_u, d_base, dstep, astep, idesc);
                        else if (ntl == 3) issue_ksteps<3>(ksl, qs, q1, a_d0, bd, ks_u, d_base, dstep, astep, idesc);
                        else if (ntl == 4) issue_ksteps<4>(ksl, qs, q1, a_d0, bd, ks_u, d_base, dstep, astep, idesc);
                        else
                            for (int q = qs; q < q1; q++, bd += ks_u) issue(a_d0 + (ksl[q] & 0xFFFFu), 1u);
                    }
                    ptx::mma_commit_elect(&sh.wempty[st]);
                }
                ptx::mma_commit_elect(&sh.in_empty[s]);
            }
            ptx::mma_commit_elect(&sh.acc_full[a]);
            __syncwarp();
        }
        if (p.prof && lane == 0) {
            unsigned long long *r = p.prof + (size_t)blockIdx.x * 32;
            r[6] = wdesc; r[7] = wacc; r[8] = win; r[9] = wwt; r[10] = clock64() - t_start; r[15] = wfence;
        }
    } else {
        // ------------------------------------------------------------------ epilogue
        const int ew = warp - kEpi0;
        unsigned long long wed = 0, wea = 0, web = 0, wtm = 0, wit = 0, wpub = 0, ntask = 0, ncomp = 0;
        const unsigned long long t_start = clock64();
        const int quad = warp % 4;        // TMEM lane quadrant this warp may access
        const int rank = ew / 4;          // (EPIW / 4) warps per quadrant split the (tile, column batch) items
        const uint32_t tmem_base = sh.tmem_base;
        for (uint32_t seq = 0;; seq++) {
            pwait(p, &sh.desc_full[seq % kRing], (seq / kRing) & 1, wed);
            const int l = sh.desc_l[seq % kRing];
            const long long t = sh.desc_t[seq % kRing];
            if (l < 0) break;
            const LayerP &L = p.layer[l];
            const Tile T = make_tile(p, l, t);
            const int a = seq % p.nacc;
            pwait(p, &sh.acc_full[a], (seq / p.nacc) & 1, wea);
            ptx::tc_fence_after();
            const int CB = L.Nc >= 32 ? 32 : 16;
            const int ncb = L.Nc / CB;
            const int Tdv = STK ? L.Td : 1;          // output planes per task (stacked 3-D layers)
            const int items = L.ntl * ncb * Tdv;
            const __nv_bfloat16 *resp = reinterpret_cast<const __nv_bfloat16 *>(L.res.ptr);
            __nv_bfloat16 *outp = reinterpret_cast<__nv_bfloat16 *>(L.out.ptr);
            uint64_t pol_keep, pol_stream;
            asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_keep));
            asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_stream));
            const int d = T.d;
            __nv_bfloat16 *scr = T.dst_scr ? reinterpret_cast<__nv_bfloat16 *>(scr_slot(p, T.slot) + L.scr_off) : nullptr;
            if (L.pool) {
                // fused max-pool (the subgraph's last layer, L620-626): per channel batch, every epilogue warp turns its
                // TMEM rows into bf16 conv outputs (bias -> ReLU -> RNE, the conv layer's own epilogue) in a shared
                // staging tile; then the 512 threads take the max over each pool window of the tile's conv positions
                // that lie inside the conv output (out-of-range taps ignored) and store the pooled
                // 16-B channel vectors.  The conv output itself is never written to global memory.
                uint4 *stg = reinterpret_cast<uint4 *>(smem + p.pool_off);
                const int nck = CB / 8;
                // channel batches staged together: the 4 warp ranks share ntl x gcb (tile, batch) items, so every
                // epilogue warp reads TMEM even when a task has a single M tile; staging <= ntl*128 x 128 ch
                const int gcb = pool_gcb(ncb, L.ntl, EPIW / 4);
                const int nchk = gcb * nck;   // 16-B chunks per staged position (a power of two)
                for (int cb0 = 0; cb0 < ncb; cb0 += gcb) {
                    const int ng = min(gcb, ncb - cb0);
                    for (int it = rank; it < L.ntl * ng; it += (EPIW / 4)) {
                        const int tl = it / ng, cbl = it - tl * ng;
                        const int ch0 = T.nc * L.Nc + (cb0 + cbl) * CB;
                        const int m = tl * 128 + quad * 32 + lane;
                        // one coalesced bias load per item (lane c holds channel ch0 + c), issued before the TMEM load;
                        // lanes take their channels' values by shuffle
                        const bool bsm = p.bias_off >= 0;   // shared bias table (warp-uniform)
                        const float bl = bsm ? 0.f : __ldg(L.bias + ch0 + (lane & (CB - 1)));
                        const float4 *bsv = reinterpret_cast<const float4 *>(smem + p.bias_off) + ((L.bofs + ch0) >> 2);
                        uint32_t r[2][16];
                        const uint32_t taddr =
                            tmem_base + a * p.acc_stride + ((uint32_t)(quad * 32) << 16) + tl * L.Nc + (cb0 + cbl) * CB;
                        ptx::tmem_ld16(taddr, r[0]);
                        if (CB == 32) ptx::tmem_ld16(taddr + 16, r[1]);
                        ptx::tmem_ld_wait();
                        ptx::reg_fence16(r[0]);
                        ptx::reg_fence16(r[1]);
#pragma unroll
                        for (int k = 0; k < 4; k++) {
                            if (k >= nck) break;
                            float v[8];
#pragma unroll
                            for (int e = 0; e < 8; e++) v[e] = __uint_as_float(r[k / 2][(k % 2) * 8 + e]);
                            if (bsm) {
                                const float4 b0 = bsv[2 * k], b1 = bsv[2 * k + 1];
                                v[0] += b0.x; v[1] += b0.y; v[2] += b0.z; v[3] += b0.w;
                                v[4] += b1.x; v[5] += b1.y; v[6] += b1.z; v[7] += b1.w;
                            } else {
#pragma unroll
                                for (int e = 0; e < 8; e++) v[e] += __shfl_sync(0xffffffffu, bl, k * 8 + e);
                            }
#pragma unroll
                            for (int e = 0; e < 8; e++)
                                if (L.relu) v[e] = fmaxf(v[e], 0.f);
                            stg[m * nchk + ((cbl * nck + k) ^ (m & (nchk - 1)))] =
                                make_uint4(pack2(v[0], v[1]), pack2(v[2], v[3]), pack2(v[4], v[5]), pack2(v[6], v[7]));
                        }
                    }
                    asm volatile("bar.sync 2, %0;" ::"n"(32 * EPIW) : "memory");
                    const int nc_g = ng * nck;                // (a power of two unless the last, partial group)
                    const int lnc = 31 - __clz(nc_g);
                    const int nout = L.Tpb * L.Tpw * nc_g;
                    for (int q = ew * 32 + lane; q < nout; q += 32 * EPIW) {
                        const int ck = (nc_g & (nc_g - 1)) ? q % nc_g : q & (nc_g - 1);
                        const int o = (nc_g & (nc_g - 1)) ? q / nc_g : q >> lnc;
                        const int oy = o / L.Tpw, ox = o - oy * L.Tpw;
                        const int py = T.py0 + oy, px = T.px0 + ox;
                        if (d >= T.hi[0] || py >= T.hi[1] || px >= T.hi[2]) continue;
                        if (p.padded && (py < T.dlo[1] || px < T.dlo[2])) continue;
                        uint4 *dst = reinterpret_cast<uint4 *>(outp + pix_pow2(L.out, L.lB, T.n, d, py, px) + T.nc * L.Nc +
                                                               cb0 * CB) + ck;
                        if (d >= L.pout[0] || py >= L.pout[1] || px >= L.pout[2]) {   // masked position of the bricked grid
                            *dst = make_uint4(0, 0, 0, 0);
                            continue;
                        }
                        // the window's taps inside the conv output (out-of-range taps ignored; pad < k keeps
                        // at least one): bounds hoisted out of the tap loops, the max starts from -inf
                        const int i0 = oy * L.ps[0], j0 = ox * L.ps[1];
                        const int rlo = max(0, -(T.y0 + i0)), rhi = min(L.pk[0], L.out_ext[1] - (T.y0 + i0));
                        const int clo = max(0, -(T.x0 + j0)), chi = min(L.pk[1], L.out_ext[2] - (T.x0 + j0));
                        const __nv_bfloat162 ninf = __halves2bfloat162(__ushort_as_bfloat16((unsigned short)0xFF80),
                                                                       __ushort_as_bfloat16((unsigned short)0xFF80));
                        __nv_bfloat162 mx[4] = {ninf, ninf, ninf, ninf};
                        for (int rr = rlo; rr < rhi; rr++) {
                            const int mrow = (i0 + rr) * L.Wp + j0;
                            for (int cc = clo; cc < chi; cc++) {
                                const int m = mrow + cc;
                                const uint4 u = stg[m * nchk + (ck ^ (m & (nchk - 1)))];
                                const __nv_bfloat162 *h = reinterpret_cast<const __nv_bfloat162 *>(&u);
                                mx[0] = __hmax2(mx[0], h[0]); mx[1] = __hmax2(mx[1], h[1]);
                                mx[2] = __hmax2(mx[2], h[2]); mx[3] = __hmax2(mx[3], h[3]);
                            }
                        }
                        *dst = *reinterpret_cast<const uint4 *>(mx);
                    }
                    asm volatile("bar.sync 2, %0;" ::"n"(32 * EPIW) : "memory");   // staging reused by the next group
                }
            }
            PT(const unsigned long long ti0 = p.prof ? clock64() : 0;)
            for (int it = rank; it < (L.pool ? 0 : items); it += (EPIW / 4)) {
                const int o = STK ? it / (L.ntl * ncb) : 0, itr = it - o * (L.ntl * ncb);   // output plane of the task
                const int tl = itr / ncb, cb = itr - tl * ncb;
                const int m = tl * 128 + quad * 32 + lane;
                const int i = m / L.Wp, j = m - i * L.Wp;
                const int y = T.y0 + i, x = T.x0 + j;
                const int d = T.d + o;
                int kind = 0;   // 0 skip, 1 zero (masked), 2 value
                if (i < L.Tb && j < L.Tw && d < T.hi[0] && y < T.hi[1] && x < T.hi[2] && (!p.padded || x >= T.dlo[2]))
                    kind = (d < L.out_ext[0] && y < L.out_ext[1] && x < L.out_ext[2]) ? 2 : 1;
                const int ch0 = T.nc * L.Nc + cb * CB;
                // global reads ahead of their use: one coalesced bias load per item (lane c holds channel ch0 + c,
                // shuffled out below) and the residual one 16-B chunk ahead (issued before the store of the previous
                // chunk, which the compiler may not move it past).  Measured on B200 against per-chunk bias loads and
                // in-order residual loads: cfg4 11.46 -> 11.25 ms, cfg3 7.28 -> 7.16 ms; all four residual chunks up
                // front (registers), two chunks ahead, or 16-channel items with the next item's reads in flight were slower.
                const bool bsm = p.bias_off >= 0;   // (warp-uniform)
                const float bl = DBG(p, 8) || bsm ? 0.f : __ldg(L.bias + ch0 + (lane & (CB - 1)));
                const float4 *bsv = reinterpret_cast<const float4 *>(smem + p.bias_off) + ((L.bofs + ch0) >> 2);
                const bool has_rs = L.has_res && kind == 2 && !DBG(p, 16);
                const uint4 *rsp = has_rs ? reinterpret_cast<const uint4 *>(resp + pix_pow2(L.res, L.lB, T.n, d, y, x) + ch0) : nullptr;
                uint32_t rnext[8] = {0, 0, 0, 0, 0, 0, 0, 0};   // residual: 16 channels per 256-bit load, one pair ahead
                if (has_rs) ld_cg_v8(rsp, rnext);
                uint32_t r[2][16];
                const uint32_t taddr = tmem_base + a * p.acc_stride + ((uint32_t)(quad * 32) << 16) +
                                       tl * (Tdv * L.Nc) + (Tdv - 1 - o) * L.Nc + cb * CB;
                PT(const unsigned long long tt0 = p.prof ? clock64() : 0;)
                ptx::tmem_ld16(taddr, r[0]);
                if (CB == 32) ptx::tmem_ld16(taddr + 16, r[1]);
                ptx::tmem_ld_wait();
                ptx::reg_fence16(r[0]);
                ptx::reg_fence16(r[1]);
                PT(if (p.prof) wtm += clock64() - tt0;)
                if (!__any_sync(0xffffffffu, kind != 0)) continue;   // (warp-uniform: the bias shuffles need every lane)
                uint4 *dst = reinterpret_cast<uint4 *>(
                    T.dst_scr ? scr + ((((long long)(d - T.dlo[0]) * L.pR[1] + (y - T.dlo[1])) * L.pR[2] + (x - T.dlo[2])) *
                                           L.cout + ch0)
                              : outp + pix_pow2(L.out, L.lB, T.n, d, y, x) + ch0);
                // 16 channels (32 B: one full sector) per 256-bit store (kind 1: zeros)
#pragma unroll
                for (int k2 = 0; k2 < 2; k2++) {
                    if (k2 >= CB / 16) break;
                    uint32_t w8[8], rr[8];
#pragma unroll
                    for (int e = 0; e < 8; e++) rr[e] = rnext[e];
                    if (has_rs && k2 + 1 < CB / 16) ld_cg_v8(rsp + 2 * (k2 + 1), rnext);   // next pair in flight
#pragma unroll
                    for (int h = 0; h < 2; h++) {   // 16-B chunk k = 2 k2 + h: channels 8k .. 8k + 7
                        const int k = 2 * k2 + h;
                        float v[8];
#pragma unroll
                        for (int e = 0; e < 8; e++) v[e] = __uint_as_float(r[k2][h * 8 + e]);
                        if (bsm) {   // shared bias table: two broadcast 16-B reads per 8 channels
                            const float4 b0 = bsv[2 * k], b1 = bsv[2 * k + 1];
                            v[0] += b0.x; v[1] += b0.y; v[2] += b0.z; v[3] += b0.w;
                            v[4] += b1.x; v[5] += b1.y; v[6] += b1.z; v[7] += b1.w;
                        } else {
#pragma unroll
                            for (int e = 0; e < 8; e++) v[e] += __shfl_sync(0xffffffffu, bl, k * 8 + e);
                        }
                        if (has_rs) {
                            const __nv_bfloat162 *h2 = reinterpret_cast<const __nv_bfloat162 *>(&rr[h * 4]);
#pragma unroll
                            for (int e = 0; e < 4; e++) {
                                const float2 f = __bfloat1622float2(h2[e]);
                                v[2 * e] += f.x;
                                v[2 * e + 1] += f.y;
                            }
                        }
                        if (L.relu) {
#pragma unroll
                            for (int e = 0; e < 8; e++) v[e] = fmaxf(v[e], 0.f);
                        }
#pragma unroll
                        for (int e = 0; e < 4; e++) w8[h * 4 + e] = kind == 2 ? pack2(v[2 * e], v[2 * e + 1]) : 0u;
                    }
                    if (kind && !DBG(p, 4)) {
                        if (L.l2hint) st_v8_pol(dst + 2 * k2, w8, L.l2hint == 1 ? pol_keep : pol_stream);
                        else st_v8(dst + 2 * k2, w8);
                    }
                }
            }
            PT(if (p.prof) { wit += clock64() - ti0; ntask++; })
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&sh.acc_empty[a]);
            // every epilogue warp's stores of this tile precede the publication
            const unsigned long long tb0 = p.prof ? clock64() : 0;
            asm volatile("bar.sync 2, %0;" ::"n"(32 * EPIW) : "memory");
            if (p.prof) web += clock64() - tb0;
            if (ew == 0 && lane == 0) {
                PT(const unsigned long long tp0 = p.prof ? clock64() : 0;)
                if (p.padded) {
                    // CTA-local hand-off to this CTA's loaders, which read the scratch through L2 (cp.async.cg)
                    __threadfence();
                    atomicMax_block(&sh.done_seq, (int)seq + 1);
                } else if (p.only_layer < 0) {
                    // the release store is cumulative over the epilogue warps' stores ordered before it by the named
                    // barrier (the bar.sync + st.release.gpu publication pattern; no separate membar.gl, which cost
                    // ~1 us per task: measured)
                    st_release(status_word(p, l, t), (int)(EP | 2));
                }
                ncomp++;
                PT(if (p.prof) wpub += clock64() - tp0;)
            }
        }
        if (ew == 0 && lane == 0 && ncomp) atomicAdd(&p.counters[0], ncomp);   // tasks computed by this CTA
        if (p.prof && ew == 0 && lane == 0) {
            unsigned long long *r = p.prof + (size_t)blockIdx.x * 32;
            r[11] = wed; r[12] = wea; r[13] = web; r[14] = clock64() - t_start;
            r[16] = wtm; r[17] = wit; r[18] = wpub; r[19] = ntask;
        }
    }
    ptx::tc_fence_before();
    __syncthreads();
    if (warp == kMma) ptx::tmem_dealloc(sh.tmem_base, p.tmem_cols);
    if (threadIdx.x == 0) run_exit(p.counters);
}

// weights [cout][kd][kh][kw][cin] bf16 -> [nc][kb][ks][2][Nc][8] per the layer's A mode
// stk (depth-stacked 3-D layer): per k-step q' = (rs, kk) the B operand is [2][kd * Nc][8]: the kd depth taps' weights
// side by side along N (tap a at rows [a*Nc, (a+1)*Nc)), so one MMA can feed several output planes.
__global__ void pack_gen_kernel(const __nv_bfloat16 *__restrict__ w, __nv_bfloat16 *__restrict__ out, int cout, int cin,
                                int kd, int kh, int kw, int amode, int Nc, int nkb, int nks, int stk) {
    const int NB = stk ? kd * Nc : Nc;           // B rows per k-step
    const int nq = stk ? nks / kd : nks;         // k-steps in the packed layout
    const long long total = (long long)(cout / Nc) * nkb * nq * 2 * NB * 8;
    const int taps = kd * kh * kw;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
        long long r = i;
        const int e = (int)(r % 8); r /= 8;
        int col = (int)(r % NB); r /= NB;
        const int j = (int)(r % 2); r /= 2;
        int q = (int)(r % nq); r /= nq;
        const int kb = (int)(r % nkb);
        const int nc = (int)(r / nkb);
        if (stk) {   // (q', a) -> the unstacked k-step q = q' * kd + a
            q = q * kd + col / Nc;
            col %= Nc;
        }
        int tap, ci, kk;
        if (amode == AM_SW128) { kstep_tap(q, kd, kh, kw, 4, tap, kk); ci = kb * 64 + kk * 16 + j * 8 + e; }
        else if (amode == AM_PLANES || amode == AM_SW64) {
            kstep_tap(q, kd, kh, kw, (cin + 15) / 16, tap, kk);
            ci = kk * 16 + j * 8 + e;
        }
        else {
            const int np = (kw + 1) / 2, u = q % np, ar = q / np;
            const int s = 2 * u + j;
            tap = s < kw ? ar * kw + s : -1;
            ci = e;
        }
        const int co = nc * Nc + col;
        float v = 0.f;
        if (tap >= 0 && tap < taps && ci < cin) v = __bfloat162float(w[((long long)co * taps + tap) * cin + ci]);
        out[i] = __float2bfloat16_rn(v);
    }
}

}  // namespace gen

// ------------------------------------------------------------------------------------------------ host
static bool gen_sw64_ok() {   // BDL_GEN_SW64=0: cin = 32 layers use the chunk-plane layout (A/B runs)
    static const int v = [] { const char *e = getenv("BDL_GEN_SW64"); return e ? atoi(e) : 1; }();
    return v != 0;
}
static int gen_amode(int cin) {
    if (cin <= 8) return gen::AM_PAIR;
    if (cin % 64 == 0) return gen::AM_SW128;
    if (cin == 32 && gen_sw64_ok()) return gen::AM_SW64;
    if (cin % 16 == 0 && cin < 64) return gen::AM_PLANES;
    return -1;
}

constexpr int kGenInBudget = 112 * 1024;   // input-stage ring
constexpr int kGenWStage = 32 * 1024;      // one weight stage
constexpr int kGenW = 3;                   // weight stages
constexpr double kGenTaskOverheadMmas = 96.0;   // fixed per-task cost in units of one 128-row MMA (tile model)
// Shallow-K subgraphs (FLOP-weighted mean reduction length cin * taps below this) run 2 weight stages and give the
// third to the input ring: larger input stages, larger tiles, fewer tasks, where the weights streamed per task are
// small.  Measured on B200 (same box, all plain subgraphs switched): ResNet-50 conv2_x / conv3_x subgraphs (mean K
// 340-900) 2.20 -> 2.01, 2.96 -> 2.64, 1.72 -> 1.66 ms; deep-K subgraphs lose (VGG-16 conv3-5, K 2000-4600: +4-11 %;
// ResNet-50 conv5_x +4-8 %).
constexpr double kGenShallowK = 1024.0;
// A/B knobs of the tile model (host only): BDL_GEN_OVH overrides the per-task cost; BDL_GEN_NW2 = 0 / 1 forces 3 / 2
// weight stages for plain (unstacked, pool-free) subgraphs instead of the shallow-K rule
static double gen_task_overhead() {
    static const double v = [] { const char *e = getenv("BDL_GEN_OVH"); return e ? atof(e) : kGenTaskOverheadMmas; }();
    return v;
}
static int gen_nw2() {
    static const int v = [] { const char *e = getenv("BDL_GEN_NW2"); return e ? atoi(e) : -1; }();
    return v;
}
static int gen_nw_force() {   // BDL_GEN_NW = 1..4: weight stages of every plain subgraph (A/B)
    static const int v = [] { const char *e = getenv("BDL_GEN_NW"); return e ? atoi(e) : 0; }();
    return v;
}

// BDL_GEN_STACK=0: no depth stacking (A/B runs)
static bool gen_stack_ok() {
    static const int v = [] { const char *e = getenv("BDL_GEN_STACK"); return e ? atoi(e) : 1; }();
    return v != 0;
}

// Static (tile-independent) fields of a layer.  Returns false if the layer cannot run on the kernel.
static bool gen_layer_static(const Layer &ly, int nsp, const bdl_layout &lo_out, gen::LayerP &G) {
    const bdl_layer &l = ly.L;
    if (l.kind != BDL_OP_CONV) return false;
    G.amode = gen_amode(l.cin);
    if (G.amode < 0 || l.cout % 16 != 0) return false;
    if (l.groups > 1) return false;   // grouped / depthwise: not a dense contraction (CUDA-core kernels)
    for (int d = 0; d < 3; d++) {
        G.k[d] = l.k[d];
        G.s[d] = l.stride[d];
        G.pd[d] = l.pad[d];
        G.dl[d] = l.dil[d] > 1 ? l.dil[d] : 1;
        G.ke[d] = G.dl[d] * (G.k[d] - 1) + 1;
        if (G.k[d] > 7 || (G.s[d] != 1 && G.s[d] != 2)) return false;
        if (G.dl[d] > 1 && G.s[d] != 1) return false;   // dilated layers: stride 1
        G.in_ext[d] = ly.in_ext[d + 1];
        G.out_ext[d] = ly.out_ext[d + 1];
    }
    if (nsp == 2 && (G.k[0] != 1 || G.s[0] != 1 || G.pd[0] != 0)) return false;
    if (G.s[0] != 1) return false;   // depth stride: not needed by the workloads
    G.cin = l.cin;
    G.cout = l.cout;
    G.grid[0] = (int)(lo_out.nb[1] * lo_out.Bd);
    G.grid[1] = (int)(lo_out.nb[2] * lo_out.Bh);
    G.grid[2] = (int)(lo_out.nb[3] * lo_out.Bw);
    G.Nc = l.cout <= 256 ? l.cout : 256;
    if (l.cout % G.Nc) return false;
    G.nnc = l.cout / G.Nc;
    const int taps = G.k[0] * G.k[1] * G.k[2];
    if (G.amode == gen::AM_SW128) { G.nkb = l.cin / 64; G.kc = 8; G.nks = taps * 4; G.row_u = 8; }
    else if (G.amode == gen::AM_PLANES) { G.nkb = 1; G.kc = l.cin / 8; G.nks = taps * ((l.cin + 15) / 16); G.row_u = 1; }
    else if (G.amode == gen::AM_SW64) { G.nkb = 1; G.kc = 4; G.nks = taps * 2; G.row_u = 4; }
    else { G.nkb = 1; G.kc = 1; G.nks = G.k[0] * G.k[1] * ((G.k[2] + 1) / 2); G.row_u = 1; }
    // the loader's address arithmetic uses shifts: power-of-two chunk counts and brick extents
    auto lg = [](int v) { int r = 0; while ((1 << r) < v) r++; return (1 << r) == v ? r : -1; };
    G.lkc = lg(G.kc);
    G.xal = 0;
    G.tma = 0;
    G.pxo = 0;
    G.lB[0] = lg(lo_out.Bd);
    G.lB[1] = lg(lo_out.Bh);
    G.lB[2] = lg(lo_out.Bw);
    if (G.lkc < 0 || G.lB[0] < 0 || G.lB[1] < 0 || G.lB[2] < 0) return false;
    if (G.nks > gen::kMaxKs) return false;
    const int ks_bytes = 2 * G.Nc * 16;
    G.kpw = std::max(1, std::min(G.nks, kGenWStage / ks_bytes));
    G.nws = (G.nks + G.kpw - 1) / G.kpw;
    G.idesc = ptx::idesc_bf16_f32(128, G.Nc);
    // depth stacking (3-D 3x3x3 layers of one K-block and one channel chunk, 3 Nc <= 256): the packed B of a k-step
    // holds the three depth taps side by side, in every mode (padded runs it with Td = 1)
    G.stk = 0;
    G.Td = 1;
    if (nsp == 3 && G.k[0] == 3 && G.s[0] == 1 && G.dl[0] == 1 && G.nkb == 1 && G.amode != gen::AM_PAIR &&
        3 * G.Nc <= 256 && G.nnc == 1 && gen_stack_ok()) {
        G.stk = 1;
        const int nq = G.nks / 3, ksb = 2 * 3 * G.Nc * 16;
        G.kpw = std::max(1, std::min(nq, kGenWStage / ksb));
        G.nws = (nq + G.kpw - 1) / G.kpw;
        for (int i = 0; i < 3; i++) G.idesc_s[i] = ptx::idesc_bf16_f32(128, (i + 1) * G.Nc);
    }
    G.nblk = G.s[1] * G.s[2];
    return true;
}

// Fused pool: epilogue staging tile, every M row of the conv tile x the channel batches staged together, bf16.
static int gen_pool_stage_bytes(const gen::LayerP &G, int er) {
    const int CB = G.Nc >= 32 ? 32 : 16, ncb = G.Nc / CB;
    const int gcb = gen::pool_gcb(ncb, G.ntl, er);   // channel batches staged together (epilogue)
    return G.ntl * 128 * gcb * CB * 2;
}

// Tile geometry: output tiles of Tb rows x Tw columns (Tw a multiple of walign) covering cover_h x
// cover_w positions of one plane; the best useful fraction of MMA rows that fits the shared memory.
// Fused-pool layers (G.pool): the loops run over pooled tiles Tpb x Tpw covering cover_h x cover_w pool outputs, and
// the conv tile is the region under their windows, Tb = (Tpb-1)*ps + pk (likewise Tw).
constexpr int kGenPoolStageMax = 32 * 1024;   // fused pool: largest epilogue staging tile

// Loader cost of a 1x1 stride-1 layer's stage in the tile model (MMA units per TMA box): one box per pixel row, or one
// per brick row of bricks when the tile height is a multiple of the brick height Bh (the multi-row TMA path).
static double gen_row_cost() {   // BDL_GEN_ROWC: A/B knob
    static const double v = [] { const char *e = getenv("BDL_GEN_ROWC"); return e ? atof(e) : 4.0; }();
    return v;
}
static bool gen_layer_tiles(gen::LayerP &G, int cover_h, int cover_w, int walign, int in_budget = kGenInBudget,
                            int max_td = 1, int bh = 0) {
    double best = -1e30;
    bool found = false;
    gen::LayerP cand = G;
    for (int Td = 1; Td <= (G.stk ? max_td : 1); Td *= 2)
    for (int Ub = std::min(cover_h, 32); Ub >= 1; Ub--) {
        for (int Uw = (cover_w + walign - 1) / walign * walign; Uw >= walign; Uw -= walign) {
            const int Tb = G.pool ? (Ub - 1) * G.ps[0] + G.pk[0] : Ub, Tw = G.pool ? (Uw - 1) * G.ps[1] + G.pk[1] : Uw;
            if (Tb > 64 || Tw > 256) continue;
            cand.Tb = Tb;
            cand.Tw = Tw;
            cand.Tpb = G.pool ? Ub : 0;
            cand.Tpw = G.pool ? Uw : 0;
            cand.in_rows = (Tb - 1) * G.s[1] + G.ke[1];
            cand.in_cols = (Tw - 1) * G.s[2] + G.ke[2];
            cand.Wp = (cand.in_cols + G.s[2] - 1) / G.s[2];
            cand.rb = (cand.in_rows + G.s[1] - 1) / G.s[1];
            cand.blk_px = cand.rb * cand.Wp;
            cand.plane_px = cand.nblk * cand.blk_px;
            const int M = Tb * cand.Wp;
            cand.ntl = (M + 127) / 128;
            cand.Td = Td;
            if (cand.ntl * Td * G.Nc > 256) continue;   // double-buffered accumulators (Td planes per task)
            const int npl = G.ke[0] + Td - 1;            // input planes of a task's stage
            const int max_tap = (npl - 1) * cand.plane_px + (cand.nblk - 1) * cand.blk_px +
                                ((G.ke[1] - 1) / G.s[1]) * cand.Wp + (G.ke[2] - 1) / G.s[2];
            int rows = std::max(npl * cand.plane_px, max_tap + cand.ntl * 128);
            rows = (rows + 7) / 8 * 8;
            if (G.amode == gen::AM_PLANES) rows += 1;   // odd plane stride: conflict-free loader stores
            if (G.amode == gen::AM_SW64) rows = (rows + 1 + 7) / 8 * 8;   // room for the alignment offset pxo
            cand.rowsA = rows;
            cand.stage_bytes = G.amode == gen::AM_SW128 ? rows * 128
                               : G.amode == gen::AM_SW64  ? rows * 64
                               : (G.amode == gen::AM_PLANES ? G.kc * rows * 16 : rows * 16);
            cand.stage_bytes = (cand.stage_bytes + 1023) / 1024 * 1024;
            if (cand.stage_bytes * 2 > in_budget) continue;   // two input stages at least
            if (G.pool && gen_pool_stage_bytes(cand, 3) > kGenPoolStageMax) continue;   // (fused pools: 12 warps)
            const int nty = (cover_h + Ub - 1) / Ub, ntx = (cover_w + Uw - 1) / Uw;
            // time model per plane: tasks x (MMAs per task + a fixed per-task cost), times a penalty for loaded
            // halo pixels.  The fixed cost (claim, dependency acquire, barriers, epilogue hand-off, publication)
            // was measured on B200 at ~3.7 us per task with the MMAs, loads and stores disabled (cfg5,
            // BDL_GEN_DBG=7), i.e. on the order of a hundred 128-row MMAs, so small tiles lose even when their
            // MMA rows are better used.
            const double halo = (double)cand.in_rows * cand.in_cols / ((double)Tb * Tw * G.s[1] * G.s[2]);
            double mmas = (double)cand.ntl * G.nks * G.nkb;
            if (G.stk) {
                // stacked: per k-step one MMA per input plane, of N = (number of output planes it feeds) x Nc, costed by
                // its shared-memory operand bytes relative to an N = Nc MMA (A 4 KB + B 32 B per N row)
                double w = 0;
                for (int i = 0; i < npl; i++) {
                    const int na = std::min(2, i) - std::max(0, i - Td + 1) + 1;
                    w += (4096.0 + na * G.Nc * 32.0) / (4096.0 + G.Nc * 32.0);
                }
                mmas = (double)cand.ntl * (G.nks / 3) * w;
            }
            // 1x1 stride-1 layers: TMA boxes per task (see gen_row_cost)
            double boxes = 0;
            if (bh > 0 && G.amode == gen::AM_SW128 && G.k[0] == 1 && G.k[1] == 1 && G.k[2] == 1 && G.s[1] == 1 &&
                G.s[2] == 1 && !G.pool)
                boxes = (double)G.nkb * (Tb % bh == 0 ? Tb / bh : Tb);
            // per output plane: tasks / Td
            const double cost = (double)nty * ntx / Td * (mmas + gen_task_overhead() + gen_row_cost() * boxes) *
                                (1.0 + 0.1 * (halo - 1.0));
            const double score = -cost + 1e-6 * Ub * Uw * Td;
            if (score > best) {
                best = score;
                G = cand;
                found = true;
            }
        }
    }
    return found;
}

// TMA rows for the generic kernel's stride-1 SW128 layers (BDL_GEN_TMA=0 disables, for A/B runs).
static bool gen_tma_ok() {
    static const int v = [] { const char *e = getenv("BDL_GEN_TMA"); return e ? atoi(e) : 1; }();
    return v != 0;
}
// 3x3 stride-2 layers by element-strided TMA rows (BDL_GEN_TMA3=0: cp.async, for A/B runs)
static bool gen_tma3_ok() {
    static const int v = [] { const char *e = getenv("BDL_GEN_TMA3"); return e ? atoi(e) : 1; }();
    return v != 0;
}
// 1x1 layers by one TMA box per brick row of bricks (BDL_GEN_TMA4=0: one box per pixel row, for A/B runs)
static bool gen_tma4_ok() {
    static const int v = [] { const char *e = getenv("BDL_GEN_TMA4"); return e ? atoi(e) : 1; }();
    return v != 0;
}
// Padded-mode first layer eligible for TMA rows (stride 1, swizzled A layout, 2-D or SW64 3-D)?
static bool gen_pad_tma_ok(const gen::LayerP &G, int nsp, int Bw) {
    if (!gen_tma_ok() || G.s[0] != 1 || G.s[1] != 1 || G.s[2] != 1 || Bw > 256) return false;
    if (G.amode == gen::AM_SW128) return G.k[0] == 1 && nsp == 2;
    return G.amode == gen::AM_SW64;
}

// 5-D view of a 2-D bricked bf16 tensor (identity BrickMap): (channel, x in brick, brick column, y in brick,
// brick row over (n, by)); box = 64 channels x Bw x nseg bricks x 1 x 1, 128-B swizzled (the SW128 A layout).
static bool gen_encode_row_map(CUtensorMap *tm, const TView &v, int nseg, int xstride = 1, int box_ch = 64,
                               int rows = 1) {
    static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult qr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &qr) != cudaSuccess ||
            !enc)
            return false;
    }
    const cuuint64_t px = (cuuint64_t)v.Cp * 2, brick = (cuuint64_t)v.brick_elems * 2;
    // dim 3 = row inside the brick (zin * Bh + yin: linear, stride one brick row of pixels), dim 4 = brick row
    // over (n, bz, by)
    cuuint64_t dims[5] = {(cuuint64_t)v.Cp, (cuuint64_t)v.B[3], (cuuint64_t)v.nb[3], (cuuint64_t)v.B[1] * v.B[2],
                          (cuuint64_t)v.nb[0] * v.nb[1] * v.nb[2]};
    cuuint64_t strides[4] = {px, brick, px * v.B[3], brick * v.nb[3]};
    cuuint32_t box[5] = {(cuuint32_t)box_ch, (cuuint32_t)v.B[3], (cuuint32_t)nseg, (cuuint32_t)rows, 1};
    cuuint32_t es[5] = {1, (cuuint32_t)xstride, 1, 1, 1};   // xstride 2: every other pixel of a brick row
    return enc(tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, v.ptr, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               box_ch == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Debug profiler buffer (BDL_GEN_PROF=1): 16 x u64 per CTA, zeroed before each launch.
static unsigned long long *gen_prof_buf = nullptr;
static unsigned long long *gen_prof_buffer(cudaStream_t s) {
    static const bool on = getenv("BDL_GEN_PROF") != nullptr;
    if (!on) return nullptr;
    if (!gen_prof_buf) cudaMalloc(&gen_prof_buf, 1024 * 32 * 8);
    cudaMemsetAsync(gen_prof_buf, 0, 1024 * 32 * 8, s);
    return gen_prof_buf;
}

struct GenGeom {
    gen::LayerP layer[kMaxLayers];
    int L;
    int nin, in_stride, nw, w_stride, acc_stride, nacc, tmem_cols, smem, pool_bytes, epiw;
    int PB[3], npb[3];
    long long scr_slot;
};

// Can the subgraph's trailing max-pool be fused into its last conv's epilogue?  2-D pool reading the last conv,
// no residual on that conv, and the conv's output is not needed by a later subgraph (then it is never materialized).
// Measured on B200 (VGG-16 N=128): fused pools win on convs of <= 128 channels in memoized / unmerged
// execution (stage 2: 1.27 -> 1.09 ms, stage 1 memoized 2.35 -> 2.26 ms) and lose on 256 / 512 channels (1.55 -> 1.75,
// 0.82 -> 0.93 ms) and in padded mode (2.53 -> 2.72 ms): those keep the separate vectorized pool kernel.
bool gen_pool_fused(const bdl_plan *p, const Subgraph &sg, int nconv, bool padded) {
    const int mode = p->opts.fuse_pool;   // 0 measured rule, 1 always, 2 never
    if (mode == 2 || nconv < 1 || nconv != sg.last - sg.first) return false;
    if (mode != 1 && (padded || p->layers[sg.first + nconv - 1].L.cout > 128)) return false;
    // large maps: the staging tile takes the input ring's shallow-K extra stage, and the smaller conv tiles cost more
    // than the separate pool pass (B200, VGG-16 conv1 block at 224^2: fused 2.10 vs 1.91 ms; at 112^2 fusing wins:
    // ResNet-50 stem 0.72 -> 0.62 ms, VGG-16 conv2 block 1.10 -> 0.95 ms)
    const Layer &cl = p->layers[sg.first + nconv - 1];
    if (mode != 1 && (long long)cl.out_ext[2] * cl.out_ext[3] > 112LL * 112) return false;
    const bdl_layer &pl = p->layers[sg.last].L;
    const int ci = sg.first + nconv - 1;
    if (pl.kind != BDL_OP_MAXPOOL || pl.input != ci) return false;
    if (pl.k[0] != 1 || pl.stride[0] != 1 || pl.pad[0] != 0) return false;
    for (int d = 1; d < 3; d++)
        if (pl.k[d] > 8 || pl.stride[d] < 1 || pl.stride[d] > pl.k[d] || pl.pad[d] >= pl.k[d]) return false;
    if (p->layers[ci].L.residual != BDL_NO_RESIDUAL) return false;
    for (const Tensor &t : p->tensors)
        if (t.producer == ci) return false;   // a live-out: later subgraphs read the conv output
    return true;
}

static bool gen_geometry(const bdl_plan *p, const Subgraph &sg, int nconv, bool padded, GenGeom &g) {
    memset(&g, 0, sizeof(g));
    g.L = nconv;
    const int nsp = p->in_layout.nsp;
    for (int j = 0; j < nconv; j++) {
        const Layer &ly = p->layers[sg.first + j];
        bdl_layout lo;
        bdl_layout_init(&lo, nsp, ly.out_ext[0], ly.L.cout, ly.out_ext[1], ly.out_ext[2], ly.out_ext[3],
                        p->in_layout.Bn, p->in_layout.Bd, p->in_layout.Bh, p->in_layout.Bw, BDL_BF16);
        if (!gen_layer_static(ly, nsp, lo, g.layer[j])) return false;
        g.layer[j].srcl = j < (int)sg.src_local.size() ? sg.src_local[j] : j - 1;
        g.layer[j].resl = j < (int)sg.res_local.size() ? sg.res_local[j] : -1;
        if (g.layer[j].resl >= 0 && g.layer[g.layer[j].resl].Nc != g.layer[j].Nc) return false;
    }
    const bool fused = gen_pool_fused(p, sg, nconv, padded && nconv > 1);
    // the pool's staging tile takes one weight stage's room (2 weight stages instead of 3), not input-ring room: smaller
    // input stages cost more, smaller tiles (measured on B200, VGG stage 1: 2.9 -> 3.7 ms when the ring shrank)
    // depth-stacked subgraphs (memoized geometry): Td planes per task need deeper input stages; the weight ring gives up
    // a stage for them (A/B knobs: BDL_GEN_MAXTD, BDL_GEN_STK_NW)
    static const int max_td_env = [] { const char *e = getenv("BDL_GEN_MAXTD"); return e ? atoi(e) : 4; }();
    static const int stk_nw_env = [] { const char *e = getenv("BDL_GEN_STK_NW"); return e ? atoi(e) : 2; }();
    bool any_stk = false;
    for (int j = 0; j < nconv; j++) any_stk = any_stk || g.layer[j].stk;
    const bool stk_geo = any_stk && !padded && max_td_env > 1;
    double kf = 0, f = 0;   // FLOP-weighted mean reduction length of the subgraph's convs
    for (int j = 0; j < nconv; j++) {
        const Layer &ly = p->layers[sg.first + j];
        const double K = (double)ly.L.cin / std::max(1, (int)ly.L.groups) * ly.L.k[0] * ly.L.k[1] * ly.L.k[2];
        const double F = K * ly.L.cout * ly.out_ext[1] * ly.out_ext[2] * ly.out_ext[3];
        kf += K * F;
        f += F;
    }
    const bool shallow = f > 0 && kf / f < kGenShallowK;
    // epilogue warps: 12 where the epilogue carries more per output (residual adds, depth-stacked planes), else 8 (the
    // 128 registers per thread of a 15-warp CTA).  Measured on B200 per subgraph, same box, 12 vs 8 warps: VGG-16
    // stages 1.61 / 1.55, 0.85 / 0.81, 1.21 / 1.20 ms, ResNet-50 stem 0.56 / 0.53 ms; ResNet-50 bottleneck subgraphs
    // 1.43 / 1.49, 1.62 / 1.72, 1.16 / 1.21, 0.64 / 0.69 ms; 3-D chain 1.16 / 1.25 ms.
    static const int epiw_env = [] { const char *e = getenv("BDL_GEN_EPIW"); return e ? atoi(e) : 0; }();
    bool any_res = false;
    for (int j = 0; j < nconv; j++)
        any_res = any_res || (j < (int)sg.res_tensor.size() && sg.res_tensor[j] >= 0) || g.layer[j].resl >= 0;
    g.epiw = epiw_env == 8 || epiw_env == 12 ? epiw_env : (any_res || any_stk) ? 12 : 8;
    const bool nw2 = !stk_geo && !fused && (gen_nw2() < 0 ? shallow : gen_nw2() == 1);
    const int nwp = (!stk_geo && !fused && gen_nw_force() >= 1 && gen_nw_force() <= gen::kMaxW) ? gen_nw_force()
                    : nw2 ? kGenW - 1 : kGenW;   // weight stages of a plain subgraph
    const int in_budget = stk_geo ? kGenInBudget + (kGenW - stk_nw_env) * kGenWStage
                                  : kGenInBudget + (kGenW - nwp) * kGenWStage;
    if (fused) {   // the pool's output is the last conv's task grid
        gen::LayerP &G = g.layer[nconv - 1];
        const Layer &pl = p->layers[sg.last];
        bdl_layout lp;
        bdl_layout_init(&lp, nsp, pl.out_ext[0], pl.L.cout, pl.out_ext[1], pl.out_ext[2], pl.out_ext[3], p->in_layout.Bn,
                        p->in_layout.Bd, p->in_layout.Bh, p->in_layout.Bw, BDL_BF16);
        G.pool = 1;
        for (int d = 0; d < 2; d++) {
            G.pk[d] = pl.L.k[d + 1];
            G.ps[d] = pl.L.stride[d + 1];
            G.ppd[d] = pl.L.pad[d + 1];
        }
        for (int d = 0; d < 3; d++) G.pout[d] = pl.out_ext[d + 1];
        G.grid[0] = (int)(lp.nb[1] * lp.Bd);
        G.grid[1] = (int)(lp.nb[2] * lp.Bh);
        G.grid[2] = (int)(lp.nb[3] * lp.Bw);
    }
    if (padded && nconv > 1) {
        if (!sg.chain) return false;   // padded mode: chains only (partition)
        // CTA blocks over the last layer's grid.  The planner's brick edge (rho/tau model, L649-658) sizes the
        // layout; a CTA's padded block is a band of bricks: start from the brick edge and double
        // while at least one block per SM remains, so small maps (7x7, 14x14) do not end up with 4x4 blocks whose
        // 128-row MMA tiles are mostly empty and whose halos are recomputed four times per image.
        const gen::LayerP &last = g.layer[nconv - 1];
        int B = std::max(1, sg.model_brick);
        const long long nimg = p->layers[sg.first].in_ext[0];
        auto nblocks = [&](int b) {
            long long n = nimg;
            for (int d = 0; d < 3; d++)
                if (d > 0 || nsp == 3) n *= (last.grid[d] + b - 1) / b;
            return n;
        };
        int maxg = 1;
        for (int d = 0; d < 3; d++)
            if (d > 0 || nsp == 3) maxg = std::max(maxg, last.grid[d]);
        while (B < maxg && B < 64 && nblocks(2 * B) >= (long long)p->num_sms) B *= 2;
        for (int d = 0; d < 3; d++) {
            const bool spatial = d > 0 || nsp == 3;
            g.PB[d] = spatial ? std::min(B, last.grid[d]) : 1;
            g.npb[d] = (last.grid[d] + g.PB[d] - 1) / g.PB[d];
        }
        g.scr_slot = 0;
        for (int j = 0; j < nconv; j++) {
            gen::LayerP &G = g.layer[j];
            // largest region of this layer over the blocks (the region is separable per dimension)
            for (int d = 0; d < 3; d++) {
                int mx = 0;
                for (int b = 0; b < g.npb[d]; b++) {
                    int blk[3] = {0, 0, 0}, lo[3], hi[3];
                    blk[d] = b;
                    gen::region_of(g.layer, nconv, g.PB, blk, j, lo, hi);
                    mx = std::max(mx, hi[d] - lo[d]);
                }
                G.pR[d] = std::max(1, mx);
            }
            // first layer (reads the bricked subgraph input): brick-aligned tiles so its rows arrive by TMA
            const int Bw = p->in_layout.Bw;
            const bool xal = j == 0 && gen_pad_tma_ok(G, nsp, Bw);
            G.xal = xal ? 1 : 0;
            if (!gen_layer_tiles(G, G.pR[1], xal ? G.pR[2] + Bw - 1 : G.pR[2], xal ? Bw : 1, in_budget)) return false;
            // padded sub-task ids pack (sub-tile << 8 | channel chunk): 16 + 8 bits
            const int xs = xal ? G.pR[2] + Bw - 1 : G.pR[2];
            const int tb = G.pool ? G.Tpb : G.Tb, tw = G.pool ? G.Tpw : G.Tw;
            const long long nsub = (long long)G.pR[0] * ((G.pR[1] + tb - 1) / tb) * ((xs + tw - 1) / tw);
            if (nsub >= (1LL << 16) || G.nnc >= (1 << 8)) return false;
            if (j < nconv - 1) {
                G.scr_off = g.scr_slot;
                g.scr_slot += ((long long)G.pR[0] * G.pR[1] * G.pR[2] * G.cout * 2 + 255) / 256 * 256;
            }
        }
    } else {
        for (int j = 0; j < nconv; j++) {
            gen::LayerP &G = g.layer[j];
            // pooled tiles: brick-aligned conv columns (TMA rows) when the windows tile the map (k = s, no padding)
            int walign = p->in_layout.Bw;
            if (G.pool) walign = (G.pk[1] == G.ps[1] && G.ppd[1] == 0 && p->in_layout.Bw % G.ps[1] == 0) ? p->in_layout.Bw / G.ps[1] : 1;
            if (!gen_layer_tiles(G, G.grid[1], G.grid[2], walign, in_budget, stk_geo ? max_td_env : 1,
                                 nsp == 2 && gen_tma4_ok() ? p->in_layout.Bh : 0))
                return false;
            G.ntd = (G.grid[0] + G.Td - 1) / G.Td;   // plane blocks of Td output planes
            const int tb = G.pool ? G.Tpb : G.Tb, tw = G.pool ? G.Tpw : G.Tw;   // pooled: tiles of pool outputs
            G.nty = (G.grid[1] + tb - 1) / tb;
            G.ntx = (G.grid[2] + tw - 1) / tw;
            G.ntasks = (long long)p->layers[sg.first + j].out_ext[0] * G.ntd * G.nty * G.ntx * G.nnc;
            if (G.ntasks >= (1LL << gen::kTaskBits)) return false;   // order entries: (layer << 26) | task
        }
    }
    int in_stride = 0, w_stride = 0, acc = 0;
    g.pool_bytes = 0;
    for (int j = 0; j < nconv; j++) {
        const gen::LayerP &G = g.layer[j];
        in_stride = std::max(in_stride, G.stage_bytes);
        w_stride = std::max(w_stride, G.kpw * 2 * (G.stk ? 3 : 1) * G.Nc * 16);
        acc = std::max(acc, G.ntl * G.Td * G.Nc);
        if (G.pool) g.pool_bytes = (gen_pool_stage_bytes(G, g.epiw / 4) + 1023) / 1024 * 1024;
    }
    g.in_stride = in_stride;
    g.w_stride = (w_stride + 1023) / 1024 * 1024;
    g.nin = std::min(gen::kMaxIn, in_budget / in_stride);
    g.nw = g.pool_bytes ? kGenW - 1 : stk_geo ? stk_nw_env : nwp;
    if (g.pool_bytes > kGenWStage) return false;
    g.acc_stride = acc;
    g.nacc = 2 * acc <= 512 ? 2 : 1;
    g.tmem_cols = 32;
    while (g.tmem_cols < g.nacc * acc) g.tmem_cols *= 2;
    g.smem = g.nin * in_stride + g.nw * g.w_stride + g.pool_bytes + 1024;
    return g.nin >= 2 && g.smem <= 227 * 1024 - (int)sizeof(gen::Shared) - 1024;
}

// Number of leading conv layers of subgraph sg the generic kernel runs (a trailing pool runs after it
// on the CUDA-core layer kernel), or 0 if it cannot run the subgraph (in every mode).
int gen_conv_layers(const bdl_plan *p, const Subgraph &sg) {
    if (p->in_layout.dtype != BDL_BF16 || p->in_layout.Bn != 1) return 0;
    int L = sg.last - sg.first + 1;
    if (p->layers[sg.last].L.kind == BDL_OP_MAXPOOL) L--;
    if (L < 1 || L > kMaxLayers) return 0;
    for (int j = 0; j < L; j++) {
        if (p->layers[sg.first + j].L.kind != BDL_OP_CONV || p->layers[sg.first + j].L.transposed) return 0;
        const bool res = p->layers[sg.first + j].L.residual != BDL_NO_RESIDUAL;
        if (res && sg.res_tensor[j] < 0 && sg.res_local[j] < 0) return 0;
    }
    if (L < sg.last - sg.first + 1 && p->layers[sg.last].L.input != sg.first + L - 1) return 0;   // pool tail: last conv
    GenGeom g;
    if (!gen_geometry(p, sg, L, false, g)) return 0;
    if (L > 1 && sg.chain && !gen_geometry(p, sg, L, true, g)) return 0;
    return L;
}

// Can layer `li` of the plan run on the generic kernel (the planner's test for branched subgraphs)?
bool gen_layer_supported(const bdl_plan *p, int li) {
    if (p->in_layout.dtype != BDL_BF16 || p->in_layout.Bn != 1) return false;
    const Layer &ly = p->layers[li];
    if (ly.L.transposed) return false;   // transposed convs: CUDA-core brick kernels
    bdl_layout lo;
    bdl_layout_init(&lo, p->in_layout.nsp, ly.out_ext[0], ly.L.cout, ly.out_ext[1], ly.out_ext[2], ly.out_ext[3],
                    p->in_layout.Bn, p->in_layout.Bd, p->in_layout.Bh, p->in_layout.Bw, BDL_BF16);
    gen::LayerP G;
    memset(&G, 0, sizeof(G));
    return gen_layer_static(ly, p->in_layout.nsp, lo, G) && gen_layer_tiles(G, G.grid[1], G.grid[2], p->in_layout.Bw);
}

// Tasks (memo status words) of conv layer j of the generic kernel's subgraph.
int64_t gen_layer_tasks(const bdl_plan *p, const Subgraph &sg, int j) {
    const int L = gen_conv_layers(p, sg);
    if (j >= L) return 0;
    GenGeom g;
    gen_geometry(p, sg, L, false, g);
    return g.layer[j].ntasks;
}

// Padded-mode scratch: two region slots per CTA.
int64_t gen_scratch_bytes(const bdl_plan *p, const Subgraph &sg) {
    const int L = gen_conv_layers(p, sg);
    if (L <= 1) return 0;
    GenGeom g;
    gen_geometry(p, sg, L, true, g);
    return (int64_t)p->num_sms * 2 * g.scr_slot;
}

size_t gen_packed_bytes(const bdl_plan *p, const Subgraph &sg, int j) {
    const int L = gen_conv_layers(p, sg);
    if (j >= L) return 0;
    GenGeom g;
    gen_geometry(p, sg, L, false, g);
    const gen::LayerP &G = g.layer[j];
    return (size_t)G.nnc * G.nkb * G.nks * 2 * G.Nc * 8 * 2;
}

// Memo task order (host, uploaded at prepare).  Tickets are drawn along it; any order is correct (the scheduler
// claims missing dependencies first), the order only decides locality and waiting.
//  * default: locality-aware wavefront (the paper's future work, L1785-1791).  Images run in groups large
//    enough to keep every SM busy; inside a group each task gets a scan key: a task that reads only external
//    tensors is keyed by the fraction of its input frame (d, y, x raster order) its window reaches, and a task
//    with producers inside the subgraph by the largest key among its dependencies plus a lag of about two
//    waves of that layer's tasks.  Sorting by key interleaves the layers as a wavefront that streams each image
//    top to bottom: a layer's tiles are consumed shortly after they are produced, while they are still in L2,
//    instead of layer by layer (3-D volumes: 402 MB of cfg5 intermediates would not fit).
//  * schedule_seed != 0: a seeded random topological order (Kahn's algorithm drawing uniformly from the ready
//    set), for schedule-invariance tests.
std::vector<int> gen_task_order(const bdl_plan *p, const Subgraph &sg) {
    const int L = gen_conv_layers(p, sg);
    std::vector<int> ord;
    if (L <= 0) return ord;
    GenGeom g;
    gen_geometry(p, sg, L, false, g);
    const int N = p->layers[sg.first].in_ext[0];
    std::vector<long long> base(L + 1, 0);
    for (int j = 0; j < L; j++) base[j + 1] = base[j] + g.layer[j].ntasks;
    const long long total = base[L];
    auto enc = [&](int j, long long t) { return (j << gen::kTaskBits) | (int)t; };
    if (p->opts.schedule_seed) {
        // dependents lists + in-degrees, then Kahn with a seeded uniform pick from the ready set
        std::vector<int> indeg(total, 0);
        std::vector<std::vector<int>> out(total);
        for (int j = 0; j < L; j++)
            for (long long t = 0; t < g.layer[j].ntasks; t++) {
                const gen::Deps D = gen::deps_of(g.layer, j, t);
                for (int i = 0; i < D.ns + D.nr; i++) {
                    int dl;
                    const long long dt = gen::dep_at(g.layer, D, i, dl);
                    out[base[dl] + dt].push_back((int)(base[j] + t));
                    indeg[base[j] + t]++;
                }
            }
        std::vector<int> ready;
        for (long long u = 0; u < total; u++)
            if (!indeg[u]) ready.push_back((int)u);
        std::mt19937 rng((unsigned)p->opts.schedule_seed);
        while (!ready.empty()) {
            const size_t k = std::uniform_int_distribution<size_t>(0, ready.size() - 1)(rng);
            const int u = ready[k];
            ready[k] = ready.back();
            ready.pop_back();
            const int j = (int)(std::upper_bound(base.begin(), base.end(), (long long)u) - base.begin()) - 1;
            ord.push_back(enc(j, u - base[j]));
            for (int v : out[u])
                if (--indeg[v] == 0) ready.push_back(v);
        }
        return ord;
    }
    static const bool layer_major = [] { const char *e = getenv("BDL_GEN_ORDER"); return e && !strcmp(e, "layer"); }();
    long long per_img0 = g.layer[0].ntasks / N;
    // images per group: the group's first layer holds `group_waves` waves of tasks (enough ready work at every
    // dependency level; measured on B200, cfg4: 2 waves 13.3 ms, 4 waves 11.6 ms, 8 waves 11.2 ms)
    const double gw = p->opts.group_waves > 0 ? p->opts.group_waves : 8.0;
    // lag of a consumer layer behind its producers, in waves of its tasks (BDL_GEN_LAGWAVES: A/B knob); measured on
    // B200 (r02e build): 1 / 2 / 3 / 4 / 6 waves: VGG-16 7.72 / 6.18 / 6.06 / 6.01 / 6.00 ms, ResNet-50 7.67 / 7.59 /
    // 7.59 / 7.58 / 7.56 ms, 3-D 1.37 / 1.25 / 1.25 / 1.25 / 1.25 ms.  3-D volumes keep 2: their longer lag's footprint
    // outgrows L2 (ncu, 128^3 x 32: gen_kernel DRAM reads 197 MB at 2 waves, 433 MB at 4, same time)
    static const double lw_env = [] { const char *e = getenv("BDL_GEN_LAGWAVES"); return e ? atof(e) : 0.0; }();
    const double lw = lw_env > 0 ? lw_env : p->in_layout.nsp == 3 ? 2.0 : 4.0;
    int G = (int)std::max<long long>(1, (long long)std::ceil(gw * p->num_sms / std::max<long long>(1, per_img0)));
    G = std::min(G, N);
    std::vector<double> key(total, 0.0);
    for (int j = 0; j < L; j++) {
        const gen::LayerP &C = g.layer[j];
        const double per_img = (double)C.ntasks / N;
        // BDL_GEN_ORDER=layer (A/B runs): layer by layer inside each image group
        const double lag = layer_major ? 2.0 : std::min(1.0, lw * p->num_sms / (G * per_img));
        const double frame = (double)C.in_ext[0] * C.in_ext[1] * C.in_ext[2];
        for (long long t = 0; t < C.ntasks; t++) {
            const gen::Deps D = gen::deps_of(g.layer, j, t);
            double k = -1.0;
            for (int i = 0; i < D.ns + D.nr; i++) {
                int dl;
                const long long dt = gen::dep_at(g.layer, D, i, dl);
                k = std::max(k, key[base[dl] + dt]);
            }
            if (D.ns == 0) {   // reads an external tensor: how far down its input frame the window reaches
                const gen::TaskC c = gen::decode(C, t);
                const int z = std::min(C.in_ext[0] - 1, (c.d * C.Td + C.Td - 1) * C.s[0] - C.pd[0] + C.ke[0] - 1);
                const int y = std::min(C.in_ext[1] - 1, (gen::tile_y0(C, c.ty) + C.Tb - 1) * C.s[1] - C.pd[1] + C.ke[1] - 1);
                const int x = std::min(C.in_ext[2] - 1, (gen::tile_x0(C, c.tx) + C.Tw - 1) * C.s[2] - C.pd[2] + C.ke[2] - 1);
                k = std::max(k, ((double)std::max(z, 0) * C.in_ext[1] + std::max(y, 0)) * C.in_ext[2] + std::max(x, 0)) /
                    frame;
            }
            if (D.ns + D.nr > 0) k += lag;
            key[base[j] + t] = k;
        }
    }
    struct E { int grp; double key; int j; long long t; };
    std::vector<E> es;
    es.reserve(total);
    for (int j = 0; j < L; j++) {
        const long long per = g.layer[j].ntasks / N;
        for (long long t = 0; t < g.layer[j].ntasks; t++) es.push_back({(int)(t / per) / G, key[base[j] + t], j, t});
    }
    std::stable_sort(es.begin(), es.end(), [](const E &a, const E &b) {
        if (a.grp != b.grp) return a.grp < b.grp;
        if (a.key != b.key) return a.key < b.key;
        return a.j < b.j;
    });
    for (const E &e : es) ord.push_back(enc(e.j, e.t));
    return ord;
}

bdl_status launch_pack_gen(const bdl_plan *p, const Subgraph &sg, int j, void *w_out, cudaStream_t s) {
    const int L = gen_conv_layers(p, sg);
    GenGeom g;
    gen_geometry(p, sg, L, false, g);   // packing depends only on the static fields
    const gen::LayerP &G = g.layer[j];
    const bdl_layer &l = p->layers[sg.first + j].L;
    const long long total = (long long)G.nnc * G.nkb * G.nks * 2 * G.Nc * 8;
    const int grid = (int)std::min<long long>((total + 255) / 256, 4096);
    gen::pack_gen_kernel<<<grid, 256, 0, s>>>((const __nv_bfloat16 *)l.w, (__nv_bfloat16 *)w_out, l.cout, l.cin, l.k[0],
                                              l.k[1], l.k[2], G.amode, G.Nc, G.nkb, G.nks, G.stk);
    BDL_CUDA_CHECK_LAUNCH("pack_gen");
    return BDL_OK;
}

bdl_status launch_brick_subgraph(bdl_plan *p, const Subgraph &sg, const TView &in, const TView &out,
                                 const std::vector<TView> &res_views, unsigned char *ws, cudaStream_t s, int *launches);

bdl_status launch_gen_subgraph(bdl_plan *p, Subgraph &sg, const std::vector<TView> &srcv, const TView &out,
                               const std::vector<TView> &res, unsigned char *wsp, cudaStream_t s, int *launches) {
    const int L = gen_conv_layers(p, sg);
    if (L <= 0) return fail(BDL_EUNSUPPORTED, "generic tcgen05 kernel: subgraph not supported");
    const bool padded = sg.mode == BDL_MODE_PADDED && L > 1;
    const bool pool_fused = gen_pool_fused(p, sg, L, padded);
    const bool pool_tail = L < sg.last - sg.first + 1 && !pool_fused;
    GenGeom g;
    gen_geometry(p, sg, L, padded, g);
    gen::Params P;
    memset(&P, 0, sizeof(P));
    P.L = L;
    P.prof = gen_prof_buffer(s);
#ifdef BDL_DEBUG   // timing knobs that deliberately skip work (wrong results): debug builds only
    if (const char *e = getenv("BDL_GEN_DBG")) P.dbg = atoi(e);
#endif
    if (getenv("BDL_GEN_GEOM")) {
        for (int j = 0; j < L; j++) {
            const gen::LayerP &G = g.layer[j];
            fprintf(stderr, "gen sg[%d..%d] layer %d: cin %d cout %d amode %d Tb %d Tw %d Wp %d ntl %d Nc %d nnc %d nkb %d nks %d kpw %d nws %d "
                    "in_rows %d in_cols %d rowsA %d stage %d ntasks %lld | nin %d nw %d w_stride %d smem %d padded %d\n",
                    sg.first, sg.last, j, G.cin, G.cout, G.amode, G.Tb, G.Tw, G.Wp, G.ntl, G.Nc, G.nnc, G.nkb, G.nks, G.kpw,
                    G.nws, G.in_rows, G.in_cols, G.rowsA, G.stage_bytes, G.ntasks, g.nin, g.nw, g.w_stride, g.smem, (int)padded);
        }
    }
    const int nsp = p->in_layout.nsp;
    std::vector<TView> outs(L);
    for (int j = 0; j < L; j++) {
        const Layer &ly = p->layers[sg.first + j];
        gen::LayerP &G = P.layer[j];
        G = g.layer[j];
        if (j == L - 1 && !pool_tail) {
            outs[j] = out;
        } else {
            bdl_layout lo;
            bdl_layout_init(&lo, nsp, ly.out_ext[0], ly.L.cout, ly.out_ext[1], ly.out_ext[2], ly.out_ext[3],
                            p->in_layout.Bn, p->in_layout.Bd, p->in_layout.Bh, p->in_layout.Bw, BDL_BF16);
            outs[j] = make_view(lo, wsp + sg.memo_off[j]);
        }
        G.src = G.srcl >= 0 ? outs[G.srcl] : srcv[j];
        G.out = outs[j];
        {   // L2 policy of the epilogue stores (locality-aware memoization; BDL_GEN_L2HINT=0 turns it off)
            static const int hint = [] { const char *e = getenv("BDL_GEN_L2HINT"); return e ? atoi(e) : 1; }();
            bool read_inside = false;
            for (int q = j + 1; q < L; q++)
                read_inside = read_inside || (q < (int)sg.src_local.size() ? sg.src_local[q] : q - 1) == j ||
                              (q < (int)sg.res_local.size() && sg.res_local[q] == j);
            G.l2hint = !hint || padded ? 0 : read_inside ? 1 : 2;
        }
        G.tma = 0;
        G.pxo = 0;
        // pooled tiles start at tx * Tpw * ps - pad: TMA rows need that brick-aligned and non-negative
        const bool pool_al = !G.pool || (G.ppd[0] == 0 && G.ppd[1] == 0 && (G.Tpw * G.ps[1]) % p->in_layout.Bw == 0);
        // (padded mode: only the first layer, whose tiles are brick-aligned (xal); later layers read CTA scratch)
        const int Bh = p->in_layout.Bh;
        if (!pool_al) {
        } else if (!padded && G.amode == gen::AM_SW128 && G.k[0] == 1 && G.k[1] == 1 && G.k[2] == 1 && G.s[1] == 1 &&
                   G.s[2] == 1 && G.pd[1] == 0 && G.pd[2] == 0 && nsp == 2 && !G.pool && !G.src.bmap &&
                   G.Wp == G.Tw && G.Tb % Bh == 0 && G.Tw % p->in_layout.Bw == 0 && G.Tw / p->in_layout.Bw <= 256 &&
                   Bh <= 256 && G.src.Cp % 64 == 0 && gen_tma_ok() && gen_tma4_ok() &&
                   gen_encode_row_map(&P.tm_row[j], G.src, G.Tw / p->in_layout.Bw, 1, 64, Bh)) {
            G.tma = 4;   // 1x1 stride-1 layer, brick-row-aligned tiles: one TMA box per Bh rows (the brick's rows)
        } else if ((!padded || G.xal) && G.amode == gen::AM_SW128 && G.s[1] == 1 && G.s[2] == 1 && G.k[0] == 1 && nsp == 2 &&
            !G.src.bmap && G.Tw % p->in_layout.Bw == 0 && G.Tw / p->in_layout.Bw <= 256 && G.src.Cp % 64 == 0 &&
            gen_tma_ok() && gen_encode_row_map(&P.tm_row[j], G.src, G.Tw / p->in_layout.Bw))
            G.tma = 1;
        else if ((!padded || G.xal) && G.amode == gen::AM_SW64 && G.s[0] == 1 && G.s[1] == 1 && G.s[2] == 1 && !G.src.bmap &&
                 G.Tw % p->in_layout.Bw == 0 && G.Tw / p->in_layout.Bw <= 256 && G.src.Cp == 32 &&
                 G.Wp % 2 == 0 && G.plane_px % 2 == 0 && p->in_layout.Bd * p->in_layout.Bh <= 256 && gen_tma_ok() &&
                 gen_encode_row_map(&P.tm_row[j], G.src, G.Tw / p->in_layout.Bw, 1, 32)) {
            // TMA destinations must be 128-B aligned: with even row pitches, shift the stage by one 64-B row when
            // the first in-tile column (pd) is odd
            G.tma = 1;
            G.pxo = G.pd[2] & 1;
        }
        else if (!padded && G.amode == gen::AM_SW128 && G.k[0] == 1 && G.k[1] == 1 && G.k[2] == 1 && G.s[1] == 2 &&
                 G.s[2] == 2 && G.pd[1] == 0 && G.pd[2] == 0 && nsp == 2 && !G.src.bmap && p->in_layout.Bw % 2 == 0 &&
                 G.Tw % p->in_layout.Bw == 0 && 2 * G.Tw / p->in_layout.Bw <= 256 && G.src.Cp % 64 == 0 &&
                 gen_tma_ok() && gen_encode_row_map(&P.tm_row[j], G.src, 2 * G.Tw / p->in_layout.Bw, 2))
            G.tma = 2;
        else if (!padded && G.amode == gen::AM_SW128 && G.k[0] == 1 && G.ke[1] == 3 && G.ke[2] == 3 && G.s[1] == 2 &&
                 G.s[2] == 2 && G.pd[1] == 1 && G.pd[2] == 1 && nsp == 2 && !G.src.bmap && G.Tw % p->in_layout.Bw == 0 &&
                 2 * G.Tw / p->in_layout.Bw <= 256 && G.src.Cp % 64 == 0 && gen_tma_ok() && gen_tma3_ok() &&
                 gen_encode_row_map(&P.tm_row[j], G.src, 2 * G.Tw / p->in_layout.Bw, 2))
            G.tma = 3;   // 3x3 stride-2 rows: two element-strided TMA boxes (even / odd columns) per input row
        G.has_res = sg.res_tensor[j] >= 0 || G.resl >= 0;
        if (getenv("BDL_GEN_GEOM"))
            fprintf(stderr, "gen sg[%d..%d] layer %d: tma %d amode %d s %d,%d k %d,%d Tb %d Tw %d nkb %d\n", sg.first, sg.last, j,
                    G.tma, G.amode, G.s[1], G.s[2], G.k[1], G.k[2], G.Tb, G.Tw, G.nkb);
        if (sg.res_tensor[j] >= 0) G.res = res[j];
        else if (G.resl >= 0) G.res = outs[G.resl];
        G.relu = ly.L.relu;
        G.w = (const __nv_bfloat16 *)(wsp + (ly.gen_w_off >= 0 ? ly.gen_w_off : ly.tc_w_off));
        G.bias = (const float *)(wsp + ly.b_off);
        G.task_base = sg.task_base[j];
    }
    P.nin = g.nin;
    P.pool_off = g.nin * g.in_stride + g.nw * g.w_stride;
    // fp32 bias table in the shared memory left over (BDL_GEN_BIAS_SMEM=0: A/B knob, per-item global loads)
    int smem_launch = g.smem;
    {
        static const int bias_env = [] { const char *e = getenv("BDL_GEN_BIAS_SMEM"); return e ? atoi(e) : 1; }();
        int bt = 0;
        for (int j = 0; j < L; j++) {
            P.layer[j].bofs = bt;
            bt += (P.layer[j].cout + 3) / 4 * 4;
        }
        const int boff = (P.pool_off + g.pool_bytes + 15) / 16 * 16;
        const int need = boff + bt * 4 + 1024;   // (+ the 1024-B alignment slack of g.smem)
        P.bias_off = -1;
        if (bias_env && need <= 227 * 1024 - (int)sizeof(gen::Shared) - 1024) {
            P.bias_off = boff;
            smem_launch = std::max(g.smem, need);
        }
    }
    P.in_stride = g.in_stride;
    P.nw = g.nw;
    P.w_stride = g.w_stride;
    P.nacc = g.nacc;
    P.acc_stride = g.acc_stride;
    P.tmem_cols = g.tmem_cols;
    P.status = (int *)(wsp + sg.status_off);
    P.defer = p->opts.memo_defer;
    P.counters = (unsigned long long *)(wsp + sg.counter_off);
    bool any_stk = false;
    for (int j = 0; j < L; j++) any_stk = any_stk || P.layer[j].stk;
    auto kern = any_stk ? (g.epiw == 8 ? gen::gen_kernel<true, 8> : gen::gen_kernel<true, 12>)
                        : (g.epiw == 8 ? gen::gen_kernel<false, 8> : gen::gen_kernel<false, 12>);
    const int nthreads = 32 * (gen::kEpi0 + g.epiw);
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_launch);
    const bool unmerged = sg.mode == BDL_MODE_UNMERGED || L == 1;
    if (padded) {
        P.padded = 1;
        P.only_layer = -1;
        for (int d = 0; d < 3; d++) {
            P.PB[d] = g.PB[d];
            P.npb[d] = g.npb[d];
        }
        P.scratch = wsp + sg.gen_scr_off;
        P.scr_slot = g.scr_slot;
        P.norder = (long long)p->layers[sg.first].in_ext[0] * g.npb[0] * g.npb[1] * g.npb[2];
        const int grid = (int)std::min<long long>(P.norder, p->num_sms);
        launch_pdl(kern, dim3(grid), dim3(nthreads), smem_launch, s, P);
        *launches += 1;
    } else if (!unmerged) {
        P.only_layer = -1;
        P.order = (const int *)(wsp + sg.order_off);
        P.norder = sg.norder;
        const int grid = (int)std::min<long long>(P.norder, p->num_sms);
        launch_pdl(kern, dim3(grid), dim3(nthreads), smem_launch, s, P);
        *launches += 1;
    } else {
        P.order = nullptr;
        for (int j = 0; j < L; j++) {
            P.only_layer = j;
            P.norder = P.layer[j].ntasks;
            const int grid = (int)std::min<long long>(P.norder, p->num_sms);
            launch_pdl(kern, dim3(grid), dim3(nthreads), smem_launch, s, P);
            *launches += 1;
        }
    }
    BDL_CUDA_CHECK_LAUNCH("generic tcgen05 kernel");
    if (pool_tail) {   // trailing pool: CUDA-core layer kernel on the materialized conv output
        Subgraph ps;
        ps.first = ps.last = sg.last;
        ps.mode = BDL_MODE_UNMERGED;
        ps.res_tensor = {-1};
        ps.status_off = sg.status_off;
        ps.counter_off = sg.counter_off + 64;   // the pool's own counters
        ps.task_base = {0};
        ps.scratch_off = -1;
        ps.grid = 4 * p->num_sms;
        std::vector<TView> nores(1);
        return launch_brick_subgraph(p, ps, outs[L - 1], out, nores, wsp, s, launches);
    }
    return BDL_OK;
}

int gen_launches(const bdl_plan *p, const Subgraph &sg) {
    const int L = gen_conv_layers(p, sg);
    const bool pool_tail = L < sg.last - sg.first + 1 &&
                           !gen_pool_fused(p, sg, L, sg.mode == BDL_MODE_PADDED && L > 1);
    const bool unmerged = sg.mode == BDL_MODE_UNMERGED || L == 1;
    return (unmerged ? L : 1) + (pool_tail ? 1 : 0);
}

}  // namespace bdl

// Debug: copy the generic kernel's per-CTA role profile (16 x u64 per CTA) of the last launch to host.
extern "C" int bdl_debug_gen_prof(unsigned long long *host, int max_ctas) {
    if (!bdl::gen_prof_buf) return 0;
    const int n = max_ctas < 1024 ? max_ctas : 1024;
    cudaDeviceSynchronize();
    cudaMemcpy(host, bdl::gen_prof_buf, (size_t)n * 32 * 8, cudaMemcpyDeviceToHost);
    return n;
}
