// Memo-table atomics microbenchmarks on B200 (§4.4: the A100 measurement of the cost of the
// compulsory claim / release atomics, T_atomic = 87.45 ns).  Measurement infrastructure, not
// part of the merged-execution path: built as its own library (libbdl_microbench.so) and driven by
// tools/microbench.py.
//
//   bdl_mb_cas: `ctas` CTAs x 1 thread each run `iters` dependent atomicCAS operations on a status word
//     (state 0 -> 1 -> 0 ..., each CAS's expected value comes from the previous one's result, so the latencies add):
//     mode 0 = every thread its own word (uncontended, one 128-B line per thread),
//     mode 1 = all threads one word (contended: every CAS but one per round fails),
//     mode 2 = the 3-state protocol of one memo unit: ld.acquire, CAS 0 -> 1, st.release 2 (claim + publish),
//              per thread on its own words, in sequence.
//   Reports the mean ns per operation (per CAS; per claim+publish for mode 2) from globaltimer deltas measured on
//   the device, averaged over threads.
#include <cuda_runtime.h>
#include <cstdint>

namespace {

__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ int ld_acq(const int *p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_rel(int *p, int v) {
    asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__global__ void cas_kernel(int *words, int iters, int mode, unsigned long long *ns_out, unsigned long long *fails_out) {
    int *w = mode == 1 ? words : words + blockIdx.x * 32;   // own 128-B line per thread (modes 0, 2)
    unsigned long long fails = 0;
    __syncthreads();
    const unsigned long long t0 = gtime();
    if (mode == 2) {
        for (int i = 0; i < iters; i++) {
            int *sw = w + (i & 15);               // a fresh unit of the thread's line each time
            const int epoch = (i >> 4) + 1;       // tags of the previous round read as "not started"
            const int cur = ld_acq(sw);
            const int want = epoch << 2 | 1;
            if (atomicCAS(sw, cur, want) != cur) fails++;
            st_rel(sw, epoch << 2 | 2);
        }
    } else {
        int expect = 0;
        for (int i = 0; i < iters; i++) {
            const int got = atomicCAS(w, expect, expect ^ 1);
            if (got != expect) fails++;
            expect = got ^ (got == expect ? 1 : 0);   // dependent chain: next expected value from this result
        }
    }
    const unsigned long long t1 = gtime();
    ns_out[blockIdx.x] = t1 - t0;
    fails_out[blockIdx.x] = fails;
}

}  // namespace

extern "C" int bdl_mb_cas(int ctas, int iters, int mode, double *ns_per_op, double *fail_frac) {
    int *words = nullptr;
    unsigned long long *ns = nullptr, *fl = nullptr;
    if (cudaMalloc(&words, (size_t)ctas * 32 * 4) != cudaSuccess) return 1;
    cudaMalloc(&ns, ctas * 8);
    cudaMalloc(&fl, ctas * 8);
    cudaMemset(words, 0, (size_t)ctas * 32 * 4);
    cas_kernel<<<ctas, 1>>>(words, 16, mode, ns, fl);   // warm-up (TLB, L2)
    cudaMemset(words, 0, (size_t)ctas * 32 * 4);
    cas_kernel<<<ctas, 1>>>(words, iters, mode, ns, fl);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long hns[4096], hfl[4096];
    const int n = ctas < 4096 ? ctas : 4096;
    cudaMemcpy(hns, ns, n * 8, cudaMemcpyDeviceToHost);
    cudaMemcpy(hfl, fl, n * 8, cudaMemcpyDeviceToHost);
    double s = 0, f = 0;
    for (int i = 0; i < n; i++) {
        s += (double)hns[i] / iters;
        f += (double)hfl[i] / iters;
    }
    *ns_per_op = s / n;
    *fail_frac = f / n;
    cudaFree(words);
    cudaFree(ns);
    cudaFree(fl);
    return e == cudaSuccess ? 0 : 2;
}

// ---------------------------------------------------------------------------------------------------------------------
// FFMA throughput of the device (the "alu" roofline peak of the fp32 CUDA-core paths: measured on the
// box, not derived): every thread runs 8 independent fp32 FMA chains; 4 CTAs of 256 threads per SM.
namespace {
__global__ void ffma_kernel(float *out, int iters, float a, float b) {
    float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int k = 0; k < 16; k++) {
            x0 = fmaf(x0, a, b); x1 = fmaf(x1, a, b); x2 = fmaf(x2, a, b); x3 = fmaf(x3, a, b);
            x4 = fmaf(x4, a, b); x5 = fmaf(x5, a, b); x6 = fmaf(x6, a, b); x7 = fmaf(x7, a, b);
        }
    }
    const float s = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
    if (s == 1234.5f) out[blockIdx.x] = s;   // keeps the chains live
}
}  // namespace

extern "C" int bdl_mb_ffma(double *tflops) {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float *out = nullptr;
    cudaMalloc(&out, 4096 * 4);
    const int grid = sms * 4, block = 256, iters = 4096;
    ffma_kernel<<<grid, block>>>(out, 16, 0.999f, 0.001f);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    double best = 0;
    for (int r = 0; r < 3; r++) {
        cudaEventRecord(e0);
        ffma_kernel<<<grid, block>>>(out, iters, 0.999f, 0.001f);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        const double flops = 2.0 * 8 * 16 * (double)iters * grid * block;
        best = flops / (ms * 1e-3) / 1e12 > best ? flops / (ms * 1e-3) / 1e12 : best;
    }
    *tflops = best;
    cudaFree(out);
    return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
