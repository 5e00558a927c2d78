/*
 * brickdl.h -- C ABI of the B200-native BrickDL merged conv-chain engine.
 *
 * Operations follow the paper's problem statement (PAPER.md = the ICPP'24 BrickDL paper text;
 * "L<n>" = its line numbers):
 *   - brick a tensor / unbrick it ............... §3.3.4
 *   - BrickInfo adjacency ....................... Fig 6c
 *   - partition a layer graph into subgraphs .... §3.3.1
 *   - choose padded / memoized mode (Delta rule)  §3.3.2
 *   - choose the brick size (rho / tau model) ... §3.3.3
 *   - run merged execution of a subgraph ........ §3.2; padded §3.2.1;
 *                                                  memoized §3.2.2
 *
 * Conventions (all entry points):
 *   - Every call returns bdl_status; on failure bdl_last_error() holds a thread-local message.
 *     No C++ exception crosses this boundary.
 *   - "DEVICE" pointers are CUDA global-memory pointers on the current device; "HOST" pointers
 *     are ordinary host memory.  The caller owns every buffer it passes (tensors, workspace,
 *     brick maps, weights) and the stream; the library owns only the opaque bdl_plan.
 *   - Streams are passed as `void *` holding a cudaStream_t (NULL = legacy default stream).
 *     All device work is enqueued asynchronously on that stream; no call synchronizes the device
 *     except bdl_plan_counters (which copies 32 bytes device->host).
 *   - Tensors are logical N x C x D x H x W (D = 1 for 2-D); element dtype is bdl_dtype.
 *   - A shape that is not a multiple of the brick is NOT an error: partial bricks are zero-
 *     masked (L742-743).
 */
#ifndef BRICKDL_H
#define BRICKDL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    BDL_OK = 0,
    BDL_EINVAL = 1,        /* bad shape / null pointer / brick smaller than a kernel's halo (L741) */
    BDL_EUNSUPPORTED = 2,  /* operator outside the mergeable set this build implements (L378-385) */
    BDL_ENOMEM = 3,        /* host allocation failed */
    BDL_ECUDA = 4,         /* a CUDA runtime call failed; message carries cudaGetErrorString */
    BDL_EDEADLOCK = 5      /* memo spin watchdog tripped (debug builds) */
} bdl_status;

typedef enum { BDL_F32 = 0, BDL_BF16 = 1 } bdl_dtype;

typedef enum {
    BDL_MODE_AUTO = 0,      /* the paper's static analysis decides (Delta > 15% -> memoized, L644) */
    BDL_MODE_PADDED = 1,    /* §3.2.1: each output tile recomputes its halo through the chain */
    BDL_MODE_MEMOIZED = 2,  /* §3.2.2: bricks published once to a memo table (3-state CAS tags) */
    BDL_MODE_UNMERGED = 3   /* one layer at a time (the paper's library fallback, L659-662) */
} bdl_mode;

typedef enum { BDL_OP_CONV = 0, BDL_OP_MAXPOOL = 1 } bdl_opkind;

#define BDL_NO_RESIDUAL (-2)
#define BDL_GRAPH_INPUT (-1)

/* Logical tensor + brick geometry (value type; filled by bdl_layout_init).
 * Bricked storage: physical brick p = brickmap[logical] (identity if brickmap == NULL), logical
 * index row-major over (bn, bd, bh, bw); each brick is [Bn][Bd][Bh][Bw][c_pad] row-major with
 * channels innermost (bricks block batch + spatial dims, never channels, L374-376, L738-739).
 * c_pad = C rounded up to 8 (bf16) or 4 (f32) so a pixel is a whole number of 16-byte vectors;
 * padded channels and masked positions hold zeros. */
typedef struct bdl_layout {
    int32_t nsp;                 /* 2 or 3 spatial dims */
    int32_t dtype;               /* bdl_dtype */
    int64_t N, C, D, H, W;       /* logical extents, D = 1 for 2-D */
    int32_t Bn, Bd, Bh, Bw;      /* brick extents (Bd = 1 for 2-D) */
    int32_t c_pad;               /* padded channel count */
    int32_t elem_bytes;          /* 4 (f32) or 2 (bf16) */
    int64_t nb[4];               /* bricks along n, d, h, w (ceil-div) */
    int64_t nbricks;
    int64_t brick_elems;         /* Bn*Bd*Bh*Bw*c_pad */
    int64_t brick_bytes;
    int64_t total_bytes;         /* nbricks * brick_bytes */
    const int32_t *brickmap;     /* DEVICE [nbricks] logical -> physical permutation, or NULL.
                                    Caller-owned; must outlive every call that uses the layout. */
} bdl_layout;

/* One operator of a layer graph.  Layers are listed in a topological order. */
typedef struct bdl_layer {
    int32_t kind;                /* bdl_opkind */
    int32_t cin, cout;           /* maxpool: cin == cout */
    int32_t k[3], stride[3], pad[3];  /* (d, h, w); 2-D layers use k[0] = stride[0] = 1, pad[0] = 0 */
    int32_t relu;                /* ReLU after bias (+ residual) */
    int32_t input;               /* producer layer index, or BDL_GRAPH_INPUT */
    int32_t residual;            /* BDL_NO_RESIDUAL, BDL_GRAPH_INPUT, or a layer index whose OUTPUT is
                                    added before ReLU (epilogue order bias -> residual -> ReLU) */
    const void *w;               /* DEVICE weights [cout][kd][kh][kw][cin] in the graph dtype; read only
                                    by bdl_plan_prepare (may be freed afterwards).  NULL for maxpool. */
    const float *bias;           /* DEVICE [cout] fp32 or NULL; read only by bdl_plan_prepare */
    int32_t dil[3];              /* dilation (d, h, w); <= 0 reads as 1.  Input extent of a window d(k-1)+1 (SURVEY Q19,
                                    the mergeable set of L378-385).  Tensor-core kernels: stride 1 when dilated. */
    int32_t groups;              /* <= 1: dense conv; g > 1: grouped / depthwise (g = cin) conv, weights
                                    [cout][kd][kh][kw][cin/g]; runs on the CUDA-core brick kernels (not a dense contraction) */
    int32_t transposed;          /* conv only: 1 = transposed convolution (the mergeable set of L378-385): input element
                                    i reaches outputs s*i - p + d*t through tap t (weights [cout][kd][kh][kw][cin] as above,
                                    w[co][t][ci] carrying ci to co); output extent (I-1)s - 2p + d(k-1) + 1.  groups = 1;
                                    runs on the CUDA-core brick kernels.  0 = ordinary (cross-correlation) conv. */
} bdl_layer;

/* Static-analysis knobs (§3.3); bdl_plan_opts_default gives the paper's values, except delta_threshold. */
typedef struct bdl_plan_opts {
    double delta_threshold;      /* 0.10: memoized when padding data growth Delta > 10%.  The paper uses 15%
                                    (L644, "validated on multiple NVIDIA and AMD GPU architectures"); on B200 our
                                    padded mode lost at Delta = 0.13 (VGG-16 conv1 block: 2.47 vs 2.10 ms) and tied
                                    at 0.074 and 0.  A negative value selects memoized everywhere. */
    int64_t tau;                 /* 4096: rho threshold, "tau = 2^12" (L656, printed "212") */
    int32_t bcand[4];            /* {4, 8, 16, 32} brick edge candidates (L654) */
    int64_t onchip_budget;       /* bytes a merged subgraph's footprint may use; 0 = device L2 size (L611-614) */
    int32_t force_mode;          /* bdl_mode; BDL_MODE_AUTO = the performance model */
    int32_t force_brick;         /* 0 = the rho/tau model; else this brick edge for every subgraph */
    int32_t max_subgraph_layers; /* 0 = unlimited */
    int32_t num_sms;             /* 0 = query the device */
    int32_t schedule_seed;       /* 0 = locality-aware wavefront task order; else a seeded random
                                    topological order of the memo tasks (schedule-invariance testing) */
    int32_t memo_defer;          /* generic kernel, memoized: 1 = a claimed task whose dependency is in progress
                                    elsewhere is set aside and revisited ("moves on ... revisits later", L523-525);
                                    0 = it is handed to the CTA's in-order pipeline, which waits (default: measured
                                    faster on B200) */
    int32_t group_waves;         /* generic kernel, memoized: images per task-order group sized so the group's first
                                    layer holds this many waves of tasks (0 = default 8) */
    int32_t fuse_pool;           /* generic kernel: a subgraph's trailing max-pool as the last conv's epilogue
                                    (L620-626): 0 = where measured faster on B200 (memoized / unmerged, <= 128
                                    channels), 1 = always, 2 = never (separate pool kernel) */
} bdl_plan_opts;

typedef struct bdl_plan bdl_plan;  /* opaque, library-owned host object */

/* Fill *o with the paper's defaults (see bdl_plan_opts). */
void bdl_plan_opts_default(bdl_plan_opts *o);

/* Fill *out for an N x C x D x H x W tensor in (Bn,Bd,Bh,Bw) bricks.  nsp = 2 requires D = 1 and
 * Bd = 1.  EINVAL on non-positive extents or an unknown dtype.  out->brickmap is set to NULL;
 * assign a caller-owned DEVICE permutation afterwards if wanted. */
bdl_status bdl_layout_init(bdl_layout *out, int32_t nsp, int64_t N, int64_t C, int64_t D, int64_t H,
                           int64_t W, int32_t Bn, int32_t Bd, int32_t Bh, int32_t Bw, int32_t dtype);

/* BrickInfo (Fig 6c): for each brick of ONE sample's grid (nb[1] x nb[2] x nb[3]), in
 * physical order, the physical indices of its 3^nsp - 1 logical neighbours in direction order
 * row-major over (dd, dh, dw) in {-1,0,1}^nsp minus the origin; -1 = outside the grid (a zero halo).
 * brickmap_host: HOST [nb[1]*nb[2]*nb[3]] logical -> physical, or NULL (identity).
 * adj_out: HOST, caller-allocated, [nb[1]*nb[2]*nb[3]][3^nsp - 1]. */
bdl_status bdl_brickinfo(const bdl_layout *l, const int32_t *brickmap_host, int32_t *adj_out);

/* NCDHW (dense, dtype of l) -> bricked (l->total_bytes).  src, dst DEVICE; dst fully written
 * (masked positions and padded channels = 0).  One kernel launch. */
bdl_status bdl_brickify(const bdl_layout *l, const void *src, void *dst, void *stream);

/* bricked -> NCDHW dense.  src, dst DEVICE.  One kernel launch. */
bdl_status bdl_unbrickify(const bdl_layout *l, const void *src, void *dst, void *stream);

/* Static analysis (§3.3): derive layer shapes, partition the graph into subgraphs by reverse
 * traversal (footprint <= on-chip budget, pool/reduction ends a subgraph, L603-626), choose the
 * brick size (rho/tau, L649-662), the mode (Delta, L628-647), and the kernel per subgraph.
 * layers: HOST array [nlayers] (copied; weight pointers retained until bdl_plan_prepare).
 * in: layout of the graph input (its brick fixes subgraph 0's brick).  opts NULL = defaults.
 * EUNSUPPORTED for operators this build cannot merge or run. */
bdl_status bdl_graph_partition(const bdl_layer *layers, int32_t nlayers, const bdl_layout *in,
                               const bdl_plan_opts *opts, bdl_plan **out);

int32_t bdl_plan_num_subgraphs(const bdl_plan *p);

/* Subgraph i: layers [first, last], mode (bdl_mode, never AUTO), brick edge chosen by the model
 * (rho/tau; the executed brick is the layout's), Delta (padding data growth, SURVEY Q6 reading),
 * and the executing kernel (0 = CUDA-core brick kernel, 1 = tcgen05 band kernel for C = 64/128 3x3
 * chains, 2 = generic tcgen05 kernel for every other bf16 shape). */
bdl_status bdl_plan_subgraph(const bdl_plan *p, int32_t i, int32_t *first, int32_t *last,
                             int32_t *mode, int32_t *model_brick, double *delta, int32_t *kernel);

/* Override subgraph i's mode (A/B runs).  Takes effect at the next bdl_plan_prepare. */
bdl_status bdl_plan_set_mode(bdl_plan *p, int32_t i, int32_t mode);

/* Layout of the graph output (the last layer's output, same brick as the input). */
bdl_status bdl_plan_out_layout(const bdl_plan *p, bdl_layout *out);

/* Device workspace bytes for bdl_plan_prepare / bdl_run (packed weights, inter-subgraph
 * tensors, memo buffers and status tags, scratch, counters). */
int64_t bdl_plan_workspace_bytes(const bdl_plan *p);

/* Pack weights/bias into the workspace and reset memo tags and counters.  workspace: DEVICE,
 * >= bdl_plan_workspace_bytes, 256-byte aligned, caller-owned, reused by every bdl_run. */
bdl_status bdl_plan_prepare(bdl_plan *p, void *workspace, void *stream);

/* Streams and replays: a plan's workspace (memo tables, run state) serves one stream at a time -- do not
 * run the same plan/workspace on two streams concurrently.  The per-run state (ticket counter, memo-tag
 * epoch) lives in the workspace and is advanced by the kernels themselves (the last CTA of a launch
 * rewinds the ticket and bumps the epoch), so bdl_run / bdl_run_subgraph launches may be captured in a
 * CUDA graph and replayed.  A launch that fails mid-run leaves that state undefined: call
 * bdl_plan_prepare again.
 *
 * Run subgraph i (its input/residual tensors must already hold data: for i = 0 `in_bricked`,
 * otherwise earlier subgraphs' outputs in the workspace).  in_bricked / out_bricked: DEVICE,
 * bricked per the plan's input / output layouts. */
bdl_status bdl_run_subgraph(bdl_plan *p, int32_t i, const void *in_bricked, void *out_bricked,
                            void *workspace, void *stream);

/* Run every subgraph in order: merged execution of the whole graph (a2-a7 of SURVEY §8(a)). */
bdl_status bdl_run(bdl_plan *p, const void *in_bricked, void *out_bricked, void *workspace,
                   void *stream);

/* Merged execution of the whole graph with the output written as dense NC(D)HW (out_dense: DEVICE,
 * N x C x D x H x W of the graph output, dtype of the graph).  Same work as bdl_run + bdl_unbrickify: the last
 * subgraph's epilogue writes the dense layout directly when its kernel supports it (the tcgen05 band kernel in
 * memoized / unmerged mode: unbrickify fused into the last layer's stores, L742-743), otherwise its bricked output
 * is staged in the workspace and one unbrickify launch follows. */
bdl_status bdl_run_dense(bdl_plan *p, const void *in_bricked, void *out_dense, void *workspace, void *stream);

/* Number of kernels bdl_run enqueues (for launch accounting). */
int32_t bdl_plan_launches_per_run(const bdl_plan *p);

/* Memo counters of subgraph i accumulated since bdl_plan_prepare: out[0] bricks (tasks) computed,
 * out[1] successful CAS claims, out[2] failed CAS / waits on an in-progress brick, out[3] spin polls.
 * Synchronizes `stream` (copies from the DEVICE workspace).  Compulsory atomics = 2 per brick
 * (claim + release, L528-530). */
bdl_status bdl_plan_counters(const bdl_plan *p, int32_t i, const void *workspace, void *stream,
                             uint64_t out[4]);

void bdl_plan_destroy(bdl_plan *p);

/* ---- static-analysis introspection (host only; no device needed) ---- */

/* Subgraph i's model details: Delta under the first-layer-only reading (SURVEY Q6 alternative),
 * rho of the model's brick (L653), the mode the Delta rule chose before any override, and the
 * tcgen05 band height (0 = not the band kernel). */
bdl_status bdl_plan_subgraph_model(const bdl_plan *p, int32_t i, double *delta_first, int64_t *rho,
                                   int32_t *mode_model, int32_t *tc_band);

/* 1 if subgraph i's memoized / unmerged execution runs on the CTA-pair tcgen05 kernel (C = 64 3x3 chains over
 * full-width bands: two CTAs of a cluster share one M = 256 MMA, each holding half of the output channels' weights;
 * DESIGN.md §6), 0 otherwise (or on a bad index).  Host only. */
int32_t bdl_plan_subgraph_cta_pair(const bdl_plan *p, int32_t i);

/* Region analysis (Fig 4): input-region extent of each layer of layers[first..last] for
 * one interior output brick of edge b along spatial dim `dim` (1 = d, 2 = h, 3 = w), by reverse
 * traversal I = s*(O-1) + k.  layers: HOST; ext_out: HOST [last-first+1]. */
bdl_status bdl_region_extents(const bdl_layer *layers, int32_t first, int32_t last, int32_t dim, int32_t b,
                              int64_t *ext_out);

/* Brick-size model (L649-658) for a feature map N x D x H x W (nsp spatial dims): the candidate
 * edge with the largest rho = N*prod(spatial)/B^nsp not above tau; *rho receives it.  o NULL =
 * defaults. */
int32_t bdl_model_brick(const bdl_plan_opts *o, int32_t nsp, int64_t N, int64_t D, int64_t H, int64_t W,
                        int64_t *rho);

/* Thread-local text of the last error ("" if none). */
const char *bdl_last_error(void);

/* Library version string. */
const char *bdl_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BRICKDL_H */
