// TMEM read throughput microbenchmark (B200): W warps each repeatedly tcgen05.ld 32x32b.x16 (2 KB per warp
// per load) from their lane quadrant; reports bytes per SM-cycle.  Decides whether an epilogue that reads
// 3x the accumulator columns (tap-shared N=192 MMAs) is TMEM-read bound.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "../paper_conf_icpp_lakshminarasimhan24_b200/csrc/kernels/tc_ptx.cuh"
using namespace bdl::ptx;

__global__ void tld(int iters, unsigned long long *cyc, float *sink) {
    __shared__ uint32_t tbase;
    if (threadIdx.x < 32) { tmem_alloc(&tbase, 512); tmem_relinquish(); }
    tc_fence_before(); __syncthreads(); tc_fence_after();
    const int warp = threadIdx.x / 32;
    const uint32_t ta = tbase + ((uint32_t)((warp % 4) * 32) << 16);
    float acc = 0.f;
    __syncthreads();
    unsigned long long t0 = clock64();
    for (int it = 0; it < iters; it++) {
        uint32_t r[4][16];
#pragma unroll
        for (int c = 0; c < 4; c++) tmem_ld16(ta + ((it * 64 + c * 16 + warp * 16) & 511), r[c]);
        tmem_ld_wait();
#pragma unroll
        for (int c = 0; c < 4; c++) { reg_fence16(r[c]); acc += __uint_as_float(r[c][0]) + __uint_as_float(r[c][15]); }
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    if (acc == 1234.5f) sink[0] = acc;
    tc_fence_before(); __syncthreads();
    if (threadIdx.x < 32) tmem_dealloc(tbase, 512);
}

int main() {
    unsigned long long *d; float *s;
    cudaMalloc(&d, 256 * 8); cudaMalloc(&s, 4);
    for (int w : {4, 8, 16}) {
        int iters = 4000;
        tld<<<148, 32 * w>>>(10, d, s);
        tld<<<148, 32 * w>>>(iters, d, s);
        cudaDeviceSynchronize();
        unsigned long long h; cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
        double bytes = (double)iters * 4 * 2048 * w;
        printf("warps=%2d  TMEM read %.1f B/cycle/SM  (%s)\n", w, bytes / h, cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
