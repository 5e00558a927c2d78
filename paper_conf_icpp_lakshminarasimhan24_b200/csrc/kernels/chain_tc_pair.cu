// CTA-pair tcgen05 kernel for MEMOIZED (and unmerged) merged execution of C = 64 3x3 conv chains over
// full-width bands (§3.2.2, Fig 2d; the cfg2 bench path), bf16 in / fp32 accumulate.
//
// Why a pair.  At C = 64 a single-CTA M = 128 x N = 64 x K = 16 MMA reads 4 KB of A and 2 KB of B from shared
// memory and costs 48 cycles (ideal 32: the tensor core's shared-memory operand port, ~128 B/clk, is the bound);
// the per-CTA weight ring, the epilogue staging tile and the residual tile add more shared-memory traffic
// (~73 cycles per MMA inside the single-CTA band kernel, tools/trace_ws.py).  Here two CTAs of a cluster run one
// M = 256 MMA (tcgen05 cta_group::2): each CTA supplies its own 128 A rows (its own band task) and HALF of B
// (32 of the 64 output channels), so an SM reads 4 + 1 KB per 128x64x16 (43 cycles, tools/pair_mma_test.cu), the
// halved weights of every layer stay resident (36 KB per layer per CTA: no weight streaming), and the epilogue
// writes its results straight from registers to the bricked output (one 128-B pixel per thread, 256-bit stores;
// no staging tile), reading the residual from global memory.
//
// Roles per CTA (cluster rank 0 = leader, 1 = peer), 15 warps:
//   warp 0   leader: scheduler.  Draws PAIRS of tasks (two consecutive entries of the host-built wavefront order,
//            both of one layer), claims each with the three-state CAS protocol (0 -> 1, L513-531), claims not-started
//            dependencies first (Fig 2d), and emits pair-tasks (layer, task of CTA 0, task of CTA 1; -1 = idle half)
//            into its own queue and, through DSMEM, into the peer's.
//   warp 1   loader: waits for its task's dependencies (state 2), TMA-loads the (Tb+2)-row input band (one 5-D box per
//            row) into a 128-B swizzled A buffer; rows outside the image are zero-filled.
//   warp 2   leader: MMA issuer (one elected lane, M = 256 pair MMAs, tile-outer order so the epilogue of tile t
//            overlaps the MMAs of tile t+1); peer: forwards "my tile is loaded" to the leader's barrier.
//   warps 3-14 epilogue: 4 warps (one per TMEM lane quadrant) per M tile; tcgen05.ld -> +bias (+residual) -> ReLU
//            -> bf16 -> 256-bit global stores; the CTA's 12 epilogue warps then publish the task (state 2).
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "common.cuh"
#include "tc_ptx.cuh"

namespace bdl {

namespace pr {

constexpr int C = 64;
constexpr int kQ = 4;             // scheduler -> loader queue
constexpr int kRing = 8;          // task descriptor ring (loader -> MMA / epilogue)
constexpr int kStack = 160;
constexpr int kMaxNin = 3;        // input band buffers (p.nin: 2 or 3, by geometry)
constexpr int kMaxTl = 4;         // M tiles per task
constexpr int kMaxL = 4;          // layers (resident weights)
constexpr int kEpiWarps = 12;
constexpr int kLoadWarp = 1, kMmaWarp = 2, kEpi0 = 3, kPubWarp = kEpi0 + kEpiWarps;
constexpr int kThreads = 32 * (kPubWarp + 1);
constexpr uint32_t kWLayer = 9 * 8 * 32 * 16;   // one layer's half-N weights per CTA: [tap][8 k-chunks][32 rows][16 B]
constexpr uint32_t kAccCols = 256;
constexpr int kG = 8;                           // zero guard pixels before row 0 of a band buffer (1 KB: keeps rows aligned)              // one accumulator = kMaxTl x 64 columns; two accumulators

struct Layer {
    const __nv_bfloat16 *w;   // packed [9][C/8][C][8] (launch_pack_tc)
    const float *bias;
    int relu, res;
    TView out;
};

struct Params {
    CUtensorMap tm_row[kMaxL][8];   // 5-D maps of each layer's source: box = k (1..Bh) pixel rows of one brick row x
                                    // (W/Bw + 1) bricks (the last one outside the map: zero fill) x 64 channels
    __nv_bfloat16 *dense;        // non-null: the LAST layer writes dense NCHW here (unbrickify fused, bdl_run_dense)
    int L, H, W, Tb, Wt, nty, lBh, lBw, ntl;
    int nin;                     // input band buffers (2 or 3)
    int qd;                      // scheduler queue depth (<= kQ): how far claims may run ahead of the loader
    uint32_t in_bytes;           // one input buffer (1024-B multiple)
    Layer layer[kMaxL];
    TView in, res;
    int *status;
    long long task_base[kMaxL];
    unsigned long long *counters;
    const int *order;            // (l << 24) | task, -1 = padding; consecutive entries form a pair; null = unmerged
    int norder;                  // order entries, or tasks of only_layer (unmerged)
    int only_layer;
    unsigned long long *trace;   // debug (BDL_TRACE): 12 x u64 per task, or null
    int trace_cap;
    int knob;                    // timing experiments (BDL_PAIR_KNOB, BDL_DEBUG builds only): 2 prefetch tensor maps,
                                 // 4 no proxy fence, 8 no dependency wait, 16 no band loads, 32 no MMAs
};

struct Shared {
    uint64_t q_full[kQ], q_empty[kQ];
    uint64_t ld_full[kMaxNin];      // peer: its band landed (TMA bytes + loader arrival)
    uint64_t in_full[kMaxNin];      // leader: both CTAs' bands present (leader TMA bytes + 2 arrivals)
    uint64_t in_empty[kMaxNin];     // pair MMAs of the buffer's task done (multicast commit)
    uint64_t acc_full[2][kMaxTl];
    uint64_t acc_empty[2];       // leader: 2 x kEpiWarps arrivals
    uint64_t wbar, wpeer;        // own resident weights landed; (leader) the peer's landed
    uint64_t pf_bar;             // first-band prefetch landed
    uint64_t desc_full[kRing];
    uint64_t epi_done[kRing];    // the CTA's epilogue warps have stored the slot's task (kEpiWarps arrivals)
    uint64_t pub_free[kRing];    // the publisher is done with the slot (the loader may reuse it)
    uint32_t tmem_base;
    int q_l[kQ], q_t[kQ], q_n[kQ];
    unsigned long long q_ts[kQ][4];   // debug trace (leader): ticket drawn, claimed, dependencies scanned, emitted
    int desc_l[kRing], desc_t[kRing], desc_n[kRing];
    int stk_l[kStack], stk_t[kStack];
    unsigned long long tr[kRing][13];   // [9]: emission time, [10..12] scheduler stamps   // debug trace timestamps per task slot
};

__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ int *status_word(const Params &p, int l, int t) { return p.status + p.task_base[l] + t; }
__device__ __forceinline__ int tag_state(int v, unsigned EP) { return ((v & ~3) == (int)EP) ? (v & 3) : 0; }
__device__ __forceinline__ void arrive_local(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ptx::smem_u32(bar)) : "memory");
}
// arrive on the barrier at the same offset in the leader CTA (this CTA's own when it is the leader)
__device__ __forceinline__ void arrive_leader(uint64_t *bar) { ptx::mbar_arrive_remote(ptx::mapa(ptx::smem_u32(bar), 0)); }
// the same without release semantics (no fence: the arriving thread's outstanding global stores are not waited for)
__device__ __forceinline__ void arrive_leader_relaxed(uint64_t *bar) {
    asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(ptx::mapa(ptx::smem_u32(bar), 0))
                 : "memory");
}

// M tiles a task needs: outputs m = i*Wt + j, i < rows, j < W
__device__ __forceinline__ int tiles_of(const Params &p, int t) {
    if (t < 0) return 0;
    const int ty = t % p.nty;
    const int rows = min(p.Tb, p.H - ty * p.Tb);
    return ((rows - 1) * p.Wt + p.W + 127) / 128;
}

// dependency k (0..8) of band task t: layer l-1 band (n, ty + k/3 - 1) (bands span the full width: k % 3 == 1 only)
__device__ __forceinline__ bool dep_of(const Params &p, int t, int k, int &dt) {
    if (k >= 9 || k % 3 != 1) return false;
    const int ty = t % p.nty, qy = ty + k / 3 - 1;
    if (qy < 0 || qy >= p.nty) return false;
    dt = t - ty + qy;
    return true;
}

__device__ __forceinline__ void ld_cg_v8(const void *p, uint32_t (&r)[8]) {
    asm volatile("ld.global.cg.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "l"(p));
}
__device__ __forceinline__ void st_v8(void *p, const uint32_t (&w)[8]) {
    asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3]),
                 "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7])
                 : "memory");
}
__device__ __forceinline__ uint32_t pack2(float a, float b) {
    __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<uint32_t *>(&v);
}

// ---------------------------------------------------------------------------------------------- scheduler
// Claim a memo tag (state 0 -> 1 of this launch's epoch, L513-531) with one CAS in the common case: the expected old
// value is the previous launch's "done" tag (every task ends a launch in state 2), else the value the CAS returned.
// Returns 1 = claimed by us, 0 = already claimed (state 1 or 2 of this epoch).  (The CAS needs no acquire: the
// scheduler reads no data through the tag; the loader acquires state 2 before it reads a dependency's output.)
__device__ __forceinline__ int claim(int *sw, unsigned EP) {
    int cur = EP >= 4 ? (int)((EP - 4) | 2) : 0;
    for (;;) {
        const int old = atomicCAS(sw, cur, (int)(EP | 1));
        if (old == cur) return 1;
        if (tag_state(old, EP) != 0) return 0;
        cur = old;
    }
}
__device__ __forceinline__ int ld_relaxed(const int *p) {
    int v;
    asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ void scheduler(const Params &p, Shared &sh, int e_first) {
    const int lane = threadIdx.x % 32;
    const unsigned EP = run_epoch(p.counters) << 2;
    const bool unmerged = p.only_layer >= 0;
    unsigned long long oks = 0, fails = 0;
    uint32_t qseq = 0;
    unsigned long long ts_tk = 0, ts_cl = 0, ts_dp = 0;   // debug trace
    auto emit = [&](int l, int t0, int t1) {
        const int slot = qseq % p.qd;
        if (qseq >= (uint32_t)p.qd) ptx::mbar_wait_cl(&sh.q_empty[slot], ((qseq / p.qd) - 1) & 1);
        if (lane == 0) {
            const int n = l < 0 ? 0 : max(tiles_of(p, t0), tiles_of(p, t1));
            sh.q_l[slot] = l;
            sh.q_t[slot] = t0;
            sh.q_n[slot] = n;
            if (p.trace) {
                sh.q_ts[slot][0] = ts_tk;
                sh.q_ts[slot][1] = ts_cl;
                sh.q_ts[slot][2] = ts_dp;
                sh.q_ts[slot][3] = gtime();
            }
            arrive_local(&sh.q_full[slot]);
            ptx::st_cluster_u32(ptx::mapa(ptx::smem_u32(&sh.q_l[slot]), 1), (uint32_t)l);
            ptx::st_cluster_u32(ptx::mapa(ptx::smem_u32(&sh.q_t[slot]), 1), (uint32_t)t1);
            ptx::st_cluster_u32(ptx::mapa(ptx::smem_u32(&sh.q_n[slot]), 1), (uint32_t)n);
            ptx::mbar_arrive_remote(ptx::mapa(ptx::smem_u32(&sh.q_full[slot]), 1));
        }
        __syncwarp();
        qseq++;
    };
    // Claim the not-started dependencies of one or two same-layer roots (Fig 2d), breadth first, so every stack entry
    // sits below its dependencies; emit from the top (dependencies first), pairing neighbours of one layer.
    auto expand = [&](int rl, int ra, int rb) {
        // (with two roots ra sits on top of rb, so the pair is emitted as (ra, rb): the leader gets ra -- the order entry
        // it prefetched the band of, for the static first ticket)
        if (lane == 0) {
            sh.stk_l[0] = rl;
            sh.stk_t[0] = rb >= 0 ? rb : ra;
            sh.stk_l[1] = rl;
            sh.stk_t[1] = ra;
        }
        int sp = rb >= 0 ? 2 : 1;
        for (int s = 0; s < sp; s++) {
            __syncwarp();
            const int sl = sh.stk_l[s], st = sh.stk_t[s];
            if (sl == 0) continue;
            int dt = 0, c = 0, busy = 0;
            if (dep_of(p, st, lane, dt)) {
                int *dw = status_word(p, sl - 1, dt);
                const int s2 = tag_state(ld_relaxed(dw), EP);
                if (s2 == 0 && claim(dw, EP)) c = 1;
                else if (s2 != 2) busy = 1;
            }
            const unsigned cm = __ballot_sync(0xffffffff, c);
            fails += __popc(__ballot_sync(0xffffffff, busy));
            oks += __popc(cm);
            if (c) {
                const int pos = sp + __popc(cm & ((1u << lane) - 1));
                if (pos < kStack) {
                    sh.stk_l[pos] = sl - 1;
                    sh.stk_t[pos] = dt;
                }
            }
            sp += __popc(cm);
        }
        __syncwarp();
        if (p.trace) ts_dp = gtime();
        while (sp > 0) {
            const int la = sh.stk_l[sp - 1], ta = sh.stk_t[sp - 1];
            if (sp >= 2 && sh.stk_l[sp - 2] == la) {
                const int tb = sh.stk_t[sp - 2];
                sp -= 2;
                emit(la, ta, tb);
            } else {
                sp -= 1;
                emit(la, ta, -1);
            }
        }
        __syncwarp();
    };
    if (unmerged) {   // no memo tags: tickets map to task pairs directly (drawn one ahead)
        unsigned long long tk_next = 0;
        if (lane == 0) tk_next = atomicAdd(&p.counters[4], 1ULL);
        for (;;) {
            const unsigned long long tk = __shfl_sync(0xffffffff, tk_next, 0);
            const long long e0 = 2 * (long long)tk;
            if (e0 >= p.norder) break;
            if (lane == 0) tk_next = atomicAdd(&p.counters[4], 1ULL);
            emit(p.only_layer, (int)e0, e0 + 1 < p.norder ? (int)e0 + 1 : -1);
        }
        emit(-1, -1, -1);
        return;
    }
    // Software pipeline over tickets (one global round trip per ticket in the common case): while ticket k's two
    // entries are claimed (lanes 0-1, CAS) and their dependencies' tags read speculatively (lanes 2-7), ticket k+1's
    // order entries are fetched (lanes 8-9) and ticket k+2 is drawn (lane 0).
    auto entry = [&](long long tk, int w) -> int { return 2 * tk + w < p.norder ? p.order[2 * tk + w] : -1; };
    // the first ticket of cluster c is c (its order entries were fetched before the PDL wait); the shared counter hands
    // out the rest
    const unsigned ncl = gridDim.x / 2;
    unsigned long long tkA = blockIdx.x / 2, tkB = 0;
    int e = lane < 2 ? e_first : -1;
    if (lane == 0) tkB = atomicAdd(&p.counters[4], 1ULL) + ncl;
    for (;;) {
        if (2 * (long long)tkA >= p.norder) break;
        if (p.trace) ts_tk = gtime();
        const int lr = e >= 0 ? e >> 24 : -1, tr = e >= 0 ? (e & 0xFFFFFF) : -1;   // lanes 0, 1: the roots
        const int l0 = __shfl_sync(0xffffffff, lr, 0), t0 = __shfl_sync(0xffffffff, tr, 0);
        const int l1 = __shfl_sync(0xffffffff, lr, 1), t1 = __shfl_sync(0xffffffff, tr, 1);
        // (1) issue every memory operation of this step before consuming any result
        const int pred = EP >= 4 ? (int)((EP - 4) | 2) : 0;
        int old = 0;
        if (lane < 2 && lr >= 0) old = atomicCAS(status_word(p, lr, tr), pred, (int)(EP | 1));
        int dst = 2, dl = -1, dt = -1;
        if (lane >= 2 && lane < 8) {
            const int r = (lane - 2) / 3, j = (lane - 2) % 3;
            const int rl = r ? l1 : l0, rt = r ? t1 : t0;
            if (rl > 0 && dep_of(p, rt, 3 * j + 1, dt)) {
                dl = rl - 1;
                dst = tag_state(ld_relaxed(status_word(p, dl, dt)), EP);
            }
        }
        const unsigned long long tkBv = __shfl_sync(0xffffffff, tkB, 0);
        int en = -1;
        if (lane >= 8 && lane < 10) en = entry((long long)tkBv, lane - 8);
        unsigned long long tkC = 0;
        if (lane == 0 && 2 * (long long)tkBv < p.norder) tkC = atomicAdd(&p.counters[4], 1ULL) + ncl;
        // (2) resolve the claims
        int claimed = 0;
        if (lane < 2 && lr >= 0) {
            if (old == pred) claimed = 1;
            else if (tag_state(old, EP) == 0) claimed = claim(status_word(p, lr, tr), EP);
        }
        const unsigned cm0 = __ballot_sync(0xffffffff, claimed) & 3;
        oks += __popc(cm0);
        if (p.trace) ts_cl = gtime();
        // dependency lanes of claimed roots: any not started (state 0) -> the full Fig 2d expansion
        const bool mine = lane >= 2 && lane < 8 && dl >= 0 && ((cm0 >> ((lane - 2) / 3)) & 1);
        const unsigned need = __ballot_sync(0xffffffff, mine && dst == 0);
        const unsigned busy = __ballot_sync(0xffffffff, mine && dst == 1);
        if (cm0 == 3 && l0 != l1) {
            // two layers: a separate expansion per root, the lower layer first (the higher may depend on it)
            const bool lo0 = l0 < l1;
            expand(lo0 ? l0 : l1, lo0 ? t0 : t1, -1);
            expand(lo0 ? l1 : l0, lo0 ? t1 : t0, -1);
        } else if (need) {
            if (cm0 == 3) expand(l0, t0, t1);
            else expand(cm0 & 1 ? l0 : l1, cm0 & 1 ? t0 : t1, -1);
        } else if (cm0) {
            fails += __popc(busy);
            if (p.trace) ts_dp = gtime();
            if (cm0 == 3) emit(l0, t0, t1);
            else emit(cm0 & 1 ? l0 : l1, cm0 & 1 ? t0 : t1, -1);
        }
        // (3) advance the pipeline
        tkA = tkBv;
        const int enx = __shfl_sync(0xffffffff, en, (lane & 1) + 8);
        e = lane < 2 ? enx : -1;
        tkB = tkC;
    }
    emit(-1, -1, -1);
    if (lane == 0) {
        if (oks) atomicAdd(&p.counters[1], oks);
        if (fails) atomicAdd(&p.counters[2], fails);
    }
}

// ---------------------------------------------------------------------------------------------- kernel
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1) memo_pair_kernel(const __grid_constant__ Params p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ Shared sh;
    const int warp = __shfl_sync(0xffffffff, (int)threadIdx.x / 32, 0), lane = threadIdx.x % 32;
    const uint32_t rank = ptx::cluster_rank();
    const bool leader = rank == 0;
    const unsigned long long t_entry = p.trace ? gtime() : 0;
    uint8_t *wsm = smem + p.nin * p.in_bytes;                           // resident weights [L][kWLayer]
    float *bias_s = reinterpret_cast<float *>(wsm + p.L * kWLayer);   // [L][C]
    if (ptx::smem_u32(smem) & 1023) __trap();   // 128-B swizzle atoms need 1024-B alignment
    // the kG guard pixels before row 0 of each band buffer are zero for every task (the left zero pad of the band's first
    // row; every other row's left pad is the previous row's out-of-image brick, zero-filled by TMA)
    for (int i = threadIdx.x; i < p.nin * kG * 8; i += kThreads)
        *reinterpret_cast<uint4 *>(smem + (i / (kG * 8)) * p.in_bytes + (i % (kG * 8)) * 16) = make_uint4(0, 0, 0, 0);
    for (int i = threadIdx.x; i < kRing * 13; i += kThreads) sh.tr[i / 13][i % 13] = 0;
    if (threadIdx.x == 0) {
        for (int i = 0; i < kQ; i++) {
            ptx::mbar_init(&sh.q_full[i], 1);
            ptx::mbar_init(&sh.q_empty[i], 2);   // (leader) its loader + the peer's loader
        }
        for (int i = 0; i < kMaxNin; i++) {
            ptx::mbar_init(&sh.ld_full[i], 1);
            ptx::mbar_init(&sh.in_full[i], 2);   // (leader) its loader (+ TMA bytes) + the peer's forwarder
            ptx::mbar_init(&sh.in_empty[i], 1);
        }
        for (int a = 0; a < 2; a++) {
            for (int t = 0; t < kMaxTl; t++) ptx::mbar_init(&sh.acc_full[a][t], 1);
            ptx::mbar_init(&sh.acc_empty[a], 2 * kEpiWarps);
        }
        ptx::mbar_init(&sh.wbar, 1);
        ptx::mbar_init(&sh.wpeer, 1);
        ptx::mbar_init(&sh.pf_bar, 1);
        for (int i = 0; i < kRing; i++) {
            ptx::mbar_init(&sh.desc_full[i], 1);
            ptx::mbar_init(&sh.epi_done[i], kEpiWarps);
            ptx::mbar_init(&sh.pub_free[i], 1);
        }
        ptx::fence_barrier_init();
    }
    if (warp == kMmaWarp) ptx::tmem_alloc2(&sh.tmem_base, 2 * kAccCols);   // both CTAs, same warp
    ptx::fence_proxy_async_smem();
    ptx::tc_fence_before();
    ptx::cluster_sync();   // barriers initialised in both CTAs before any remote arrival
    ptx::tc_fence_after();
    pdl_launch_dependents();
    if ((p.knob & 2) && warp == kLoadWarp) {
        for (int i = lane; i < p.L * 8; i += 32)
            asm volatile("prefetch.tensormap [%0];" ::"l"(&p.tm_row[i / 8][i % 8]) : "memory");
    }
    if (warp >= kEpi0 && warp < kPubWarp) {
        // resident weights: this CTA's 32 output channels of every layer (bulk copies of 512 B, spread over the idle
        // epilogue warps so that the loader starts on its first band at once) and the fp32 biases
        const int et = threadIdx.x - 32 * kEpi0;
        if (et == 0) ptx::mbar_arrive_expect_tx(&sh.wbar, p.L * (kWLayer + C * 4));
        asm volatile("bar.sync 2, %0;" ::"n"(32 * kEpiWarps) : "memory");
        for (int i = et; i < p.L * 72; i += 32 * kEpiWarps) {
            const int j = i / 72, r = i % 72;   // r = tap * 8 + k-chunk
            ptx::bulk_g2s(wsm + j * kWLayer + r * 512, p.layer[j].w + ((size_t)r * C + rank * 32) * 8, 512, &sh.wbar);
        }
        if (et < p.L) ptx::bulk_g2s(bias_s + et * C, p.layer[et].bias, C * 4, &sh.wbar);
    }
    // the scheduler's first ticket is static (cluster index): fetch its order entries now (written at prepare time)
    int e_first = -1, e_own = -1;
    if (warp == 0 && leader && p.only_layer < 0 && lane < 2 && (long long)blockIdx.x + lane < p.norder)
        e_first = p.order[blockIdx.x + lane];   // = order[2 * (blockIdx.x / 2) + lane] (blockIdx.x is even)
    if (warp == kLoadWarp && p.only_layer < 0 && (long long)blockIdx.x < p.norder) e_own = p.order[blockIdx.x];
    const unsigned long long t_init = p.trace ? gtime() : 0;
    // PDL: everything below may touch the previous kernel's output (subgraph input) or the memo tags
    pdl_wait();
    const unsigned long long t_pdl = p.trace ? gtime() : 0;

    const unsigned EP = run_epoch(p.counters) << 2;
    if (warp == 0) {
        if (leader) scheduler(p, sh, e_first);
    } else if (warp == kLoadWarp) {
        // ------------------------------------------------------------------ loader
        const bool unmerged = p.only_layer >= 0;
        const int R = p.Tb + 2;
        // Stage the band of task t of layer l: rows y0-1 .. y0+Tb; rows outside the image are zeros (generic proxy,
        // fenced for the tensor core); in-image rows arrive as one TMA box per run of rows inside one brick row
        // (Wt = W + Bw pixels per row: the box's last brick is outside the map and zero-filled, it is the row's right
        // and the next row's left zero pad).
        auto issue_band = [&](int l, int t, uint8_t *buf, uint64_t *bar) {
            const int ty = t % p.nty, img = t / p.nty;
            const int y0 = ty * p.Tb;
            const TView &src = l == 0 ? p.in : p.layer[l - 1].out;
            const int ya = max(y0 - 1, 0), yb = min(y0 + p.Tb, p.H - 1);   // in-image rows
            bool zeros = false;
            for (int a = 0; a < R; a++) {
                const int y = y0 - 1 + a;
                if (y >= 0 && y < p.H) continue;
                zeros = true;
                uint4 *d = reinterpret_cast<uint4 *>(buf + (size_t)(kG + a * p.Wt) * 128);
                for (int q = lane; q < p.Wt * 8; q += 32) d[q] = make_uint4(0, 0, 0, 0);
            }
            // (a shared-memory proxy fence costs ~1 us while the tensor core streams operands: only after zero rows)
            if (zeros) ptx::fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0 && (p.knob & 16)) arrive_local(bar);   // timing experiment: no band loads
            else if (lane == 0) {
                ptx::mbar_arrive_expect_tx(bar, (uint32_t)(yb - ya + 1) * p.Wt * 128);
                const int Bh = 1 << p.lBh;
                for (int y = ya; y <= yb;) {
                    const int k = min(yb + 1, (y & ~(Bh - 1)) + Bh) - y;   // rows of this brick row
                    ptx::tma_load_5d(buf + (size_t)(kG + (y - y0 + 1) * p.Wt) * 128, &p.tm_row[l][k - 1], 0, 0, 0,
                                     y & (Bh - 1), img * src.nb[2] + (y >> p.lBh), bar);
                    y += k;
                }
            }
        };
        // First-band prefetch: the first ticket of cluster c is static (c), so this CTA's first task is order entry
        // blockIdx.x; if it is a layer-0 task (no dependencies) its band is loaded now, while the scheduler claims it.
        int pf_task = -1;
        if (!unmerged && e_own >= 0 && (e_own >> 24) == 0) {
            pf_task = e_own & 0xFFFFFF;
            issue_band(0, pf_task, smem, &sh.pf_bar);
        }
        for (uint32_t seq = 0;; seq++) {
            const int slot = seq % p.qd;
            ptx::mbar_wait_cl(&sh.q_full[slot], (seq / p.qd) & 1);
            const int l = sh.q_l[slot], t = sh.q_t[slot], n = sh.q_n[slot];
            __syncwarp();
            if (lane == 0) arrive_leader(&sh.q_empty[slot]);
            const unsigned long long t_q = p.trace ? gtime() : 0;
            unsigned long long t_sch[4] = {0, 0, 0, 0};
            if (p.trace && leader)
                for (int f = 0; f < 4; f++) t_sch[f] = sh.q_ts[slot][f];
            const int b = seq % p.nin;
            uint8_t *buf = smem + b * p.in_bytes;
            uint64_t *bar = leader ? &sh.in_full[b] : &sh.ld_full[b];
            const bool work = l >= 0 && t >= 0;
            // dependencies first (state 2), then the buffer: the acquire + proxy fence overlap the wait for the buffer
            if (work && l > 0 && !unmerged && !(p.knob & 8)) {
                int dt;
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
            const unsigned long long t_dep = p.trace ? gtime() : 0;
            // the acquired data (generic-proxy stores of other CTAs) is read by TMA (async proxy)
            // (layer 0 reads the subgraph input, written by an earlier grid: no proxy fence needed)
            if (work && l > 0 && !(p.knob & 4)) asm volatile("fence.proxy.async.global;" ::: "memory");
            if (seq >= (uint32_t)p.nin) ptx::mbar_wait(&sh.in_empty[b], ((seq / p.nin) - 1) & 1);
            // the descriptor slot's previous task is published (the epilogue may run ahead of the publisher: without
            // this, a slot's epi_done could complete two phases before the publisher waits on the first)
            if (seq >= (uint32_t)kRing) ptx::mbar_wait(&sh.pub_free[seq % kRing], ((seq / kRing) - 1) & 1);
            if (lane == 0) {
                sh.desc_l[seq % kRing] = l;
                sh.desc_t[seq % kRing] = t;
                sh.desc_n[seq % kRing] = n;
                if (p.trace) {
                    sh.tr[seq % kRing][0] = t_q;
                    sh.tr[seq % kRing][1] = t_dep;
                    for (int f = 2; f < 9; f++) sh.tr[seq % kRing][f] = 0;
                    sh.tr[seq % kRing][9] = t_sch[3];
                    sh.tr[seq % kRing][10] = t_sch[0];
                    sh.tr[seq % kRing][11] = t_sch[1];
                    sh.tr[seq % kRing][12] = t_sch[2];
                }
                arrive_local(&sh.desc_full[seq % kRing]);
            }
            if (work && seq == 0 && pf_task >= 0) {
                // the first band was prefetched (static first ticket): reuse it if the queue confirms the task
                ptx::mbar_wait(&sh.pf_bar, 0);
                if (l == 0 && t == pf_task) {
                    __syncwarp();
                    if (lane == 0) arrive_local(bar);
                } else {
                    issue_band(l, t, buf, bar);
                }
                if (p.trace && lane == 0) sh.tr[seq % kRing][2] = gtime();
            } else if (work) {
                issue_band(l, t, buf, bar);
                if (p.trace && lane == 0) sh.tr[seq % kRing][2] = gtime();
            } else {
                __syncwarp();
                if (lane == 0) arrive_local(bar);
            }
            if (l < 0) break;
        }
    } else if (warp == kMmaWarp) {
        const uint32_t tmem = __shfl_sync(0xffffffff, sh.tmem_base, 0);
        if (!leader) {
            // ------------------------------------------------------------------ peer: forwarder
            ptx::mbar_wait(&sh.wbar, 0);
            if (lane == 0) arrive_leader(&sh.wpeer);
            for (uint32_t seq = 0;; seq++) {
                const int b = seq % p.nin;
                ptx::mbar_wait(&sh.ld_full[b], (seq / p.nin) & 1);
                const int l = sh.desc_l[seq % kRing];
                __syncwarp();
                if (lane == 0) arrive_leader(&sh.in_full[b]);
                if (l < 0) break;
            }
        } else {
            // ------------------------------------------------------------------ leader: MMA issuer
            ptx::mbar_wait(&sh.wbar, 0);
            ptx::mbar_wait_cl(&sh.wpeer, 0);
            constexpr uint32_t IDESC = ptx::idesc_bf16_f32(256, 64);
            const uint64_t bdesc0 = ptx::umma_desc_noswz(ptx::smem_u32(wsm), 512, 128);
            for (uint32_t seq = 0;; seq++) {
                const int b = seq % p.nin, a = seq & 1;
                ptx::mbar_wait_cl(&sh.in_full[b], (seq / p.nin) & 1);
                const int l = sh.desc_l[seq % kRing], n = sh.desc_n[seq % kRing];
                if (l < 0) break;
                const unsigned long long t_in = p.trace ? gtime() : 0;
                if (seq >= 2) ptx::mbar_wait_cl(&sh.acc_empty[a], ((seq / 2) - 1) & 1);
                ptx::tc_fence_after();
                if (p.trace && lane == 0) {
                    sh.tr[seq % kRing][3] = gtime();
                    sh.tr[seq % kRing][8] = t_in;
                }
                const uint64_t adesc = ptx::umma_desc_sw128(ptx::smem_u32(smem + b * p.in_bytes), 1024);
                const uint64_t bdesc = bdesc0 + (uint64_t)l * (kWLayer >> 4);
                const uint32_t d0 = tmem + a * kAccCols;
                for (int tl = 0; tl < n; tl++) {
                    if (!(p.knob & 32))   // timing experiment: no MMAs
#pragma unroll
                    for (int tap = 0; tap < 9; tap++) {
                        const uint32_t shift = (uint32_t)(kG + (tap / 3) * p.Wt + (tap % 3) - 1 + tl * 128);
#pragma unroll
                        for (int kk = 0; kk < 4; kk++)
                            ptx::mma2_bf16_elect(d0 + tl * 64, adesc + shift * 8 + kk * 2, bdesc + tap * 256 + kk * 64, IDESC,
                                                 (tap | kk) != 0);
                    }
                    ptx::mma2_commit_mc(&sh.acc_full[a][tl], 3);
                }
                ptx::mma2_commit_mc(&sh.in_empty[b], 3);
                if (p.trace && lane == 0) sh.tr[seq % kRing][4] = gtime();
                __syncwarp();
            }
        }
    } else if (warp < kPubWarp) {
        // ------------------------------------------------------------------ epilogue
        const int ew = warp - kEpi0, g = ew / 4, quad = warp % 4;
        const uint32_t tmem = __shfl_sync(0xffffffff, sh.tmem_base, 0);
        ptx::mbar_wait(&sh.wbar, 0);   // biases landed (with the weights)
        const int Hg = p.layer[0].out.nb[2] << p.lBh;
        const int mBh = (1 << p.lBh) - 1, mBw = (1 << p.lBw) - 1;
        uint32_t ph = 0;   // phase bit per (accumulator, tile)
        for (uint32_t seq = 0;; seq++) {
            ptx::mbar_wait(&sh.desc_full[seq % kRing], (seq / kRing) & 1);
            const int l = sh.desc_l[seq % kRing], t = sh.desc_t[seq % kRing], n = sh.desc_n[seq % kRing];
            if (l < 0) break;
            const int a = seq & 1;
            const Layer &ly = p.layer[l];
            const bool dn = p.dense != nullptr && l == p.L - 1;
            const float *bl = bias_s + l * C;
            const int img = t / p.nty, y0 = (t % p.nty) * p.Tb;
            for (int tile = g; tile < n; tile += 3) {
                const int bit = a * kMaxTl + tile;
                const int m = tile * 128 + quad * 32 + lane;
                const int i = m / p.Wt, j = m - i * p.Wt;
                const int y = y0 + i, x = j;
                int kind = 0;   // 0 skip, 1 masked (zero), 2 value
                if (t >= 0 && i < p.Tb && j < p.W && y < Hg) kind = y < p.H ? 2 : 1;
                const long long inb = (long long)(((y & mBh) << p.lBw) + (x & mBw)) * C;
                // residual pixel (128 B): requested before the accumulator wait, so its latency overlaps the MMAs
                uint32_t rr[4][8];
                const bool has_res = kind == 2 && ly.res;
                if (has_res) {
                    const long long rp = ((long long)img * p.res.nb[2] + (y >> p.lBh)) * p.res.nb[3] + (x >> p.lBw);
                    const uint8_t *rsp = reinterpret_cast<const uint8_t *>(p.res.ptr) + (rp * p.res.brick_elems + inb) * 2;
#pragma unroll
                    for (int c = 0; c < 4; c++) ld_cg_v8(rsp + c * 32, rr[c]);
                }
                ptx::mbar_wait(&sh.acc_full[a][tile], (ph >> bit) & 1);
                ph ^= 1u << bit;
                ptx::tc_fence_after();
                if (p.trace && ew == 0 && lane == 0 && tile == 0) sh.tr[seq % kRing][5] = gtime();
                if (t < 0) continue;   // idle half of the pair: nothing to store
                const long long pix = ((long long)img * ly.out.nb[2] + (y >> p.lBh)) * ly.out.nb[3] + (x >> p.lBw);
                uint8_t *dst = reinterpret_cast<uint8_t *>(ly.out.ptr) + (pix * ly.out.brick_elems + inb) * 2;
                const uint32_t taddr = tmem + a * kAccCols + tile * 64 + ((uint32_t)(quad * 32) << 16);
#pragma unroll
                for (int hf = 0; hf < 2; hf++) {   // 32 channels per TMEM load batch
                    uint32_t r[2][16];
                    ptx::tmem_ld16(taddr + hf * 32, r[0]);
                    ptx::tmem_ld16(taddr + hf * 32 + 16, r[1]);
                    ptx::tmem_ld_wait();
                    ptx::reg_fence16(r[0]);
                    ptx::reg_fence16(r[1]);
                    if (kind == 0) continue;
#pragma unroll
                    for (int cc = 0; cc < 2; cc++) {   // 16 channels: one 32-B sector
                        const int c = hf * 2 + cc;
                        uint32_t w8[8] = {0, 0, 0, 0, 0, 0, 0, 0};
                        if (kind == 2) {
                            float v[16];
#pragma unroll
                            for (int e = 0; e < 16; e += 4) {
                                const float4 bb = *reinterpret_cast<const float4 *>(bl + c * 16 + e);
                                v[e] = __uint_as_float(r[cc][e]) + bb.x;
                                v[e + 1] = __uint_as_float(r[cc][e + 1]) + bb.y;
                                v[e + 2] = __uint_as_float(r[cc][e + 2]) + bb.z;
                                v[e + 3] = __uint_as_float(r[cc][e + 3]) + bb.w;
                            }
                            if (has_res) {
#pragma unroll
                                for (int e = 0; e < 8; e++) {
                                    const float2 f = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162 *>(&rr[c][e]));
                                    v[2 * e] += f.x;
                                    v[2 * e + 1] += f.y;
                                }
                            }
                            if (ly.relu) {
#pragma unroll
                                for (int e = 0; e < 16; e++) v[e] = fmaxf(v[e], 0.f);
                            }
#pragma unroll
                            for (int e = 0; e < 8; e++) w8[e] = pack2(v[2 * e], v[2 * e + 1]);
                        }
                        if (dn) {
                            // dense NCHW output: lanes hold consecutive pixels of a row -> per channel one contiguous run
                            if (kind == 2) {
                                const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(w8);
                                __nv_bfloat16 *q = p.dense + (((long long)img * C + c * 16) * p.H + y) * p.W + x;
#pragma unroll
                                for (int e = 0; e < 16; e++)   // streaming stores: the graph output is not re-read here
                                    asm volatile("st.global.cs.b16 [%0], %1;" ::"l"(q + (long long)e * p.H * p.W),
                                                 "h"(__bfloat16_as_ushort(h[e])) : "memory");
                            }
                        } else {
                            st_v8(dst + c * 32, w8);
                        }
                    }
                }
            }
            // TMEM reads are complete (tcgen05.wait::ld): the accumulator may be overwritten, no memory fence needed
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) {
                arrive_leader_relaxed(&sh.acc_empty[a]);
                if (t >= 0) {
                    if (p.trace && ew == 0) sh.tr[seq % kRing][6] = gtime();
                    arrive_local(&sh.epi_done[seq % kRing]);   // release (CTA scope): this warp's stores, after __syncwarp
                }
            }
        }
    } else {
        // ------------------------------------------------------------------ publisher
        // Once every epilogue warp of this CTA has stored a task, publish it (memo state 2): the acquire of epi_done and
        // the cumulative release store make the 12 warps' stores visible to any CTA that acquires the tag.
        uint32_t ph = 0;
        unsigned long long computed = 0;
        for (uint32_t seq = 0;; seq++) {
            const int slot = seq % kRing;
            ptx::mbar_wait(&sh.desc_full[slot], (seq / kRing) & 1);
            const int l = sh.desc_l[slot], t = sh.desc_t[slot];
            if (l < 0) break;
            if (t < 0) {
                __syncwarp();
                if (lane == 0) arrive_local(&sh.pub_free[slot]);
                continue;
            }
            ptx::mbar_wait(&sh.epi_done[slot], (ph >> slot) & 1);
            ph ^= 1u << slot;
            if (lane == 0) {
                if (p.only_layer < 0) st_release(status_word(p, l, t), (int)(EP | 2));
                computed++;
                if (p.trace) {
                    const unsigned long long k = atomicAdd(&p.counters[7], 1ULL);
                    if (k < (unsigned long long)p.trace_cap) {
                        unsigned smid;
                        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
                        unsigned long long *rec = p.trace + k * 16;
                        rec[0] = ((unsigned long long)smid << 40) | ((unsigned long long)blockIdx.x << 8) | (unsigned)l;
                        rec[1] = (unsigned long long)t;
                        for (int f = 0; f < 7; f++) rec[2 + f] = sh.tr[slot][f];
                        rec[9] = sh.tr[slot][7];    // loader: TMA about to be issued
                        rec[10] = sh.tr[slot][8];   // MMA warp: both bands present
                        rec[11] = gtime();
                        rec[12] = sh.tr[slot][9];   // scheduler: emitted (leader)
                        rec[13] = sh.tr[slot][10];  // scheduler: ticket drawn
                        rec[14] = sh.tr[slot][11];  // scheduler: claims done
                        rec[15] = sh.tr[slot][12];  // scheduler: dependencies scanned
                    }
                }
                arrive_local(&sh.pub_free[slot]);
            }
            __syncwarp();
        }
        if (computed) atomicAdd(&p.counters[0], computed);
    }
    ptx::tc_fence_before();
    __syncthreads();
    ptx::cluster_sync();   // no remote arrival or pair MMA in flight when either CTA leaves
    if (warp == kMmaWarp) {
        ptx::tmem_relinquish2();
        ptx::tmem_dealloc2(sh.tmem_base, 2 * kAccCols);
    }
    if (p.trace && threadIdx.x == 0) {   // per-CTA record (layer 255): entry, exit
        const unsigned long long k = atomicAdd(&p.counters[7], 1ULL);
        if (k < (unsigned long long)p.trace_cap) {
            unsigned long long *rec = p.trace + k * 16;
            rec[0] = ((unsigned long long)blockIdx.x << 8) | 255u;
            rec[1] = 0;
            for (int f = 2; f < 11; f++) rec[f] = 0;
            rec[2] = t_entry;
            rec[3] = t_init;
            rec[4] = t_pdl;
            rec[11] = gtime();
        }
    }
    if (threadIdx.x == 0) run_exit(p.counters);
}

}  // namespace pr

// ------------------------------------------------------------------------------------------------ host
bool encode_rows_map_bf16(CUtensorMap *tm, const TView &v, int nseg, int rows);
unsigned long long *ws_trace_setup(unsigned char *wsp, const Subgraph &sg, cudaStream_t s, int *cap_out);

// Pair geometry for a C = 64 chain over an H x W map (full-width bands): band rows Tb, M tiles per task, input
// buffer bytes; false if the chain does not fit (W not a multiple of the brick width, too many layers for
// resident weights, ...).
bool pair_geometry(int L, int H, int W, int Bw, int N, int num_sms, int &Tb, int &ntl, int &in_bytes, int &smem, int &nin) {
    if (L < 1 || L > pr::kMaxL || W % Bw || W + Bw > 128 || num_sms < 2) return false;
    const int limit = 227 * 1024 - 4096;   // (static shared memory: the Shared block)
    const int Wt = W + Bw;
    double best = 1e30;
    bool ok = false;
    const int ncl = num_sms / 2;
    int force_tb = 0;
    if (const char *e = getenv("BDL_PAIR_TB")) force_tb = atoi(e);
    for (int tb = std::min(H, 16); tb >= 1; tb--) {
        if (force_tb && tb != force_tb) continue;
        const int m = (tb - 1) * Wt + W;
        const int nt = (m + 127) / 128;
        if (nt > pr::kMaxTl) continue;
        if ((long long)N * ((H + tb - 1) / tb) >= (1LL << 24)) continue;   // order entries: (layer << 24) | task
        const int rows = std::max(pr::kG + nt * 128 + 2 * Wt + 1, pr::kG + (tb + 2) * Wt);
        const int ib = (rows * 128 + 1023) / 1024 * 1024;
        for (int ni = pr::kMaxNin; ni >= 2; ni--) {
            const int sm = ni * ib + L * (int)pr::kWLayer + L * pr::C * 4;
            if (sm > limit) continue;
            // time model: pair-task waves x (tiles + per-task overhead of ~0.3 tile); the most band buffers that fit
            // (measured on B200 at cfg2: Tb = 6 with 2 buffers 47 us, Tb = 4 with 3 buffers 51 us)
            const long long tasks = (long long)N * ((H + tb - 1) / tb) * L;
            const long long pairs = (tasks + 1) / 2;
            const double cost = (double)((pairs + ncl - 1) / ncl) * (nt + 0.3);
            if (cost < best - 1e-9) {
                best = cost;
                Tb = tb;
                ntl = nt;
                in_bytes = ib;
                smem = sm;
                nin = ni;
                ok = true;
            }
            break;
        }
    }
    return ok;
}

bdl_status launch_pair_subgraph(const bdl_plan *p, const Subgraph &sg, const TView &in, const TView &out, const TView *res,
                                unsigned char *wsp, cudaStream_t s, int *launches, bool unmerged, void *dense) {
    const Layer &f = p->layers[sg.first];
    const int L = sg.last - sg.first + 1;
    int Tb, ntl, in_bytes, smem, nin;
    if (!pair_geometry(L, f.in_ext[2], f.in_ext[3], p->in_layout.Bw, f.in_ext[0], p->num_sms, Tb, ntl, in_bytes, smem, nin))
        return fail(BDL_EUNSUPPORTED, "tcgen05 pair kernel: geometry");
    pr::Params P;
    memset(&P, 0, sizeof(P));
    P.dense = (__nv_bfloat16 *)dense;
    P.L = L;
    P.H = f.in_ext[2];
    P.W = f.in_ext[3];
    P.Tb = Tb;
    P.Wt = P.W + p->in_layout.Bw;
    P.nty = (P.H + Tb - 1) / Tb;
    int lb = 0;
    while ((1 << lb) < p->in_layout.Bh) lb++;
    P.lBh = lb;
    lb = 0;
    while ((1 << lb) < p->in_layout.Bw) lb++;
    P.lBw = lb;
    P.ntl = ntl;
    P.in_bytes = (uint32_t)in_bytes;
    P.nin = nin;
    P.qd = pr::kQ;
    if (const char *e = getenv("BDL_PAIR_QD")) P.qd = std::max(1, std::min(pr::kQ, atoi(e)));
    P.in = in;
    if (res) P.res = *res;
    for (int j = 0; j < L; j++) {
        const Layer &ly = p->layers[sg.first + j];
        pr::Layer &T = P.layer[j];
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
        const TView &src = j == 0 ? P.in : P.layer[j - 1].out;
        for (int k = 1; k <= p->in_layout.Bh && k <= 8; k++)
            if (!encode_rows_map_bf16(&P.tm_row[j][k - 1], src, (P.W >> P.lBw) + 1, k))
                return fail(BDL_ECUDA, "cuTensorMapEncodeTiled (pair kernel row map) failed");
    }
    P.status = (int *)(wsp + sg.status_off);
    P.counters = (unsigned long long *)(wsp + sg.counter_off);
    P.trace = ws_trace_setup(wsp, sg, s, &P.trace_cap);
#ifdef BDL_DEBUG   // timing experiments, some of which skip work (wrong results): debug builds only
    if (const char *e = getenv("BDL_PAIR_KNOB")) P.knob = atoi(e);
#endif
    const long long ntiles = (long long)f.in_ext[0] * P.nty;
    auto k = pr::memo_pair_kernel;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (!unmerged) {
        P.only_layer = -1;
        P.order = (const int *)(wsp + sg.order_off);
        P.norder = (int)sg.norder;
        const long long pairs = (sg.norder + 1) / 2;
        const int grid = (int)std::min<long long>(2 * pairs, (long long)(p->num_sms & ~1));
        launch_pdl(k, dim3(grid), dim3(pr::kThreads), smem, s, P);
        *launches += 1;
    } else {
        P.order = nullptr;
        P.norder = (int)ntiles;
        const int grid = (int)std::min<long long>(2 * ((ntiles + 1) / 2), (long long)(p->num_sms & ~1));
        for (int l = 0; l < L; l++) {
            P.only_layer = l;
            launch_pdl(k, dim3(grid), dim3(pr::kThreads), smem, s, P);
            *launches += 1;
        }
    }
    BDL_CUDA_CHECK_LAUNCH("tcgen05 pair kernel");
    return BDL_OK;
}

}  // namespace bdl
