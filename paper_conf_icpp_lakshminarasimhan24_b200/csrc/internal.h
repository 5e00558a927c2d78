// Internal structures shared by the host planner (plan.cpp, run.cu) and the device kernels.
// Not part of the C ABI (include/brickdl.h is).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/brickdl.h"

namespace bdl {

constexpr int kMaxLayers = 16;   // layers per merged subgraph handled by one kernel

// Bricked tensor view (device side).  Dimension order everywhere: 0=n, 1=d, 2=h, 3=w.
struct TView {
    void *ptr;
    int ext[4];          // logical extents (N, D, H, W)
    int C, Cp;           // channels, padded channels
    int B[4];            // brick extents
    int nb[4];           // bricks per dim
    const int32_t *bmap; // logical -> physical, or null
    long long brick_elems;
};

// One layer as the CUDA-core brick kernels see it.
struct GLayer {
    int kind;            // bdl_opkind
    int cin, cout;
    int k[4], s[4], p[4];   // index 0 (batch) always k=1, s=1, p=0
    int dl[4];              // dilation (index 0 = 1)
    int groups;             // grouped conv: output channel co reads input channels of group co / (cout/groups)
    int tr;                 // transposed conv: output o gathers input i = (o + p - d*t) / s where divisible
    int in_ext[4], out_ext[4];
    int relu;
    int res_ext;         // 1: add the external residual view `res` (same extents as output)
    const float *w;      // packed [taps][cin][cout] fp32 (workspace)
    const float *bias;   // [cout] fp32 (workspace) or null
    TView res;
    TView out;           // memo buffer / subgraph output (bricked) for this layer's output
};

enum KernelKind { KERNEL_BRICK = 0, KERNEL_TC_BAND = 1, KERNEL_TC_GEN = 2 };

struct Layer {
    bdl_layer L;               // as given
    int in_ext[4], out_ext[4]; // (n, d, h, w)
    int64_t w_off = -1, b_off = -1;  // workspace offsets of packed weights / bias
    int64_t gen_w_off = -1;          // generic-kernel packed weights of a band-kernel subgraph (its padded mode)
    int64_t tc_w_off = -1;           // tcgen05 packed weights (band kernels: [tap][cin/8][cout][8];
                                     // generic kernel: [nc][kb][kstep][2][Nc][8])
};

struct Tensor {                 // materialized tensor between subgraphs
    int producer;               // layer index, -1 = graph input
    bdl_layout layout;
    int64_t ws_off;             // -1: user buffer (graph input / output)
};

struct Subgraph {
    int first, last;
    int mode;                   // bdl_mode (resolved)
    int mode_model;             // what the Delta rule chose
    int model_brick;            // rho/tau choice (edge)
    int64_t rho;
    double delta, delta_first;
    int kernel;                 // KernelKind the subgraph is able to run on
    int gen_layers = 0;         // generic tcgen05 kernel: leading conv layers it runs (a pool tail follows)
    bool gen_padded = false;    // band-kernel subgraph whose padded mode runs on the generic kernel
    int64_t gen_scr_off = -1;   // generic tcgen05 kernel, padded mode: per-CTA region scratch
    int in_tensor;              // index into Plan::tensors (the first layer's input)
    int out_tensor;
    bool chain = true;          // every layer reads the previous one (padded mode and the band / CUDA-core
                                // kernels need this; DAG subgraphs run memoized or unmerged on the generic kernel)
    std::vector<int> src_local;    // per layer: index (within the subgraph) of the layer it reads, or -1 = external
    std::vector<int> src_tensor;   // per layer: tensor index of an external input, or -1
    std::vector<int> res_local;    // per layer: index (within the subgraph) of the residual's producer, or -1
    std::vector<int> res_tensor;   // per layer in subgraph: tensor index of external residual, or -1
    // memoized mode
    std::vector<int64_t> memo_off; // per layer (except last): bricked intermediate buffer offsets (a live-out
                                   // layer's buffer is the tensor later subgraphs read)
    int64_t status_off = -1;       // int32 [L][tasks]
    std::vector<int64_t> task_base;// per layer offset into the status table (in words)
    int64_t ntasks_total = 0;
    int64_t counter_off = -1;      // uint64 run-state block (kernels/common.cuh: counters, ticket, epoch)
    // padded mode scratch (CUDA-core kernel)
    int64_t scratch_off = -1;
    int64_t scratch_slot_floats = 0;
    int grid = 0;                  // persistent grid size
    // tcgen05 band kernel parameters
    int tc_band = 0;               // band rows
    int tc_smem = 0;
    std::vector<int64_t> tc_inter_off;
    // warp-specialized memo kernel: locality-aware task order (uploaded at prepare)
    int64_t order_off = -1;
    int64_t norder = 0;
    std::vector<int> order_host;
};

}  // namespace bdl

struct bdl_plan {
    std::vector<bdl::Layer> layers;
    std::vector<bdl::Subgraph> sgs;
    std::vector<bdl::Tensor> tensors;
    bdl_layout in_layout, out_layout;
    bdl_plan_opts opts;
    int64_t ws_bytes = 0;
    int64_t final_off = 0;      // workspace: bricked graph output for bdl_run_dense's unbrickify fallback
    int num_sms = 148;
    int64_t l2_bytes = 0;
    bool prepared = false;
    void *prepared_ws = nullptr;
};

namespace bdl {
void set_error(const std::string &msg);
bdl_status fail(bdl_status s, const std::string &msg);
bool layout_valid(const bdl_layout *l);
// kernel that actually executes subgraph sg in its current mode
int effective_kernel(const Subgraph &sg);
TView make_view(const bdl_layout &l, void *ptr);
}  // namespace bdl
