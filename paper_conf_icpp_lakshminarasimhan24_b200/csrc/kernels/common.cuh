// Device helpers shared by the BrickDL kernels (product path only).
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "../internal.h"

namespace bdl {

__device__ __forceinline__ float to_f(float v) { return v; }
__device__ __forceinline__ float to_f(__nv_bfloat16 v) { return __bfloat162float(v); }
template <typename T> __device__ __forceinline__ T from_f(float v);
template <> __device__ __forceinline__ float from_f<float>(float v) { return v; }
template <> __device__ __forceinline__ __nv_bfloat16 from_f<__nv_bfloat16>(float v) { return __float2bfloat16_rn(v); }
// value after storage rounding, kept in fp32
template <typename T> __device__ __forceinline__ float store_round(float v) { return to_f(from_f<T>(v)); }

// Physical brick index of a logical brick (BrickMap, Fig 6b).
__device__ __forceinline__ long long tv_phys(const TView &v, long long logical) {
    return v.bmap ? (long long)v.bmap[logical] : logical;
}

// Element offset of channel 0 at logical position (n, d, h, w) (must be inside the bricked grid).
__device__ __forceinline__ long long tv_off(const TView &v, int n, int d, int h, int w) {
    int bn = n / v.B[0], bd = d / v.B[1], bh = h / v.B[2], bw = w / v.B[3];
    long long logical = (((long long)bn * v.nb[1] + bd) * v.nb[2] + bh) * v.nb[3] + bw;
    long long phys = tv_phys(v, logical);
    int in = (((n - bn * v.B[0]) * v.B[1] + (d - bd * v.B[1])) * v.B[2] + (h - bh * v.B[2])) * v.B[3] + (w - bw * v.B[3]);
    return phys * v.brick_elems + (long long)in * v.Cp;
}

__device__ __forceinline__ bool tv_inside(const TView &v, int n, int d, int h, int w) {
    return n >= 0 && n < v.ext[0] && d >= 0 && d < v.ext[1] && h >= 0 && h < v.ext[2] && w >= 0 && w < v.ext[3];
}

// ---- memory-model helpers for the memo table (release/acquire at GPU scope)
__device__ __forceinline__ int ld_acquire(const int *p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(int *p, int v) {
    asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// ---- per-run state of a persistent memo kernel, kept on the device (no host-side counters, so a plan's
// launches can be replayed from a CUDA graph).  Counter block of a subgraph (workspace, zeroed by
// bdl_plan_prepare):
//   [0] tasks computed  [1] successful CAS claims  [2] failed claims / busy deps  [3] spin polls
//       (accumulated since prepare, read by bdl_plan_counters)
//   [4] ticket counter of the running launch (starts at 0)
//   [5] memo-tag epoch of the running launch
//   [6] CTAs of the running launch that have exited
// A launch reads its epoch after pdl_wait(); the last CTA to exit rewinds the ticket counter and advances the
// epoch, so tags written by this launch read as state 0 ("not started") in the next one.
__device__ __forceinline__ unsigned run_epoch(const unsigned long long *c) {
    return (unsigned)*reinterpret_cast<const volatile unsigned long long *>(c + 5);
}
// Thread 0 of every CTA, after the CTA's last use of the ticket counter and of the epoch.
__device__ __forceinline__ void run_exit(unsigned long long *c) {
    __threadfence();
    if (atomicAdd(&c[6], 1ULL) == (unsigned long long)(gridDim.x * gridDim.y * gridDim.z) - 1) {
        atomicExch(&c[4], 0ULL);
        atomicExch(&c[6], 0ULL);
        __threadfence();
        atomicAdd(&c[5], 1ULL);
    }
}

// Programmatic dependent launch (PDL): a kernel launched with launch_pdl() may start while the previous
// kernel in the stream drains; it must call pdl_wait() before touching that kernel's outputs.
__device__ __forceinline__ void pdl_launch_dependents() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

template <typename Kern, typename... Args>
inline cudaError_t launch_pdl(Kern kernel, dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kernel, args...);
}

}  // namespace bdl

#define BDL_CUDA_CHECK_LAUNCH(name)                                                  \
    do {                                                                             \
        cudaError_t e__ = cudaGetLastError();                                        \
        if (e__ != cudaSuccess)                                                      \
            return ::bdl::fail(BDL_ECUDA, std::string(name) + ": " + cudaGetErrorString(e__)); \
    } while (0)
