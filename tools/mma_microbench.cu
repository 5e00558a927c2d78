// tcgen05 MMA throughput microbenchmark (B200): cycles per tcgen05.mma kind::f16, M=128, K=16, A and B
// from shared memory, one CTA per SM, whole-warp issue with an elected lane (uniform descriptors).
//   mode 0: A no-swizzle chunk planes (as the cp.async path), N in {32,64,128,256}
//   mode 1: A 128-B swizzled pixel rows (as the TMA path), N=64, tap-major order over 4 accumulators
//   mode 2: mode 1 + weights streamed per tap through a 4-stage ring by bulk copies from global
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "../paper_conf_icpp_lakshminarasimhan24_b200/csrc/kernels/tc_ptx.cuh"
using namespace bdl::ptx;

template <int N, int MODE>
__global__ void __launch_bounds__(128, 1) mma_loop(int iters, unsigned long long *cyc, const uint8_t *gw) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t done, wfull[4], wempty[4];
    __shared__ uint32_t tbase;
    for (int i = threadIdx.x * 16; i < 200 * 1024; i += 128 * 16) *(uint4 *)(smem + i) = make_uint4(0, 0, 0, 0);
    if (threadIdx.x == 0) {
        mbar_init(&done, 1);
        for (int i = 0; i < 4; i++) { mbar_init(&wfull[i], 1); mbar_init(&wempty[i], 1); }
        fence_barrier_init();
    }
    if (threadIdx.x < 32) { tmem_alloc(&tbase, 512); tmem_relinquish(); }
    fence_proxy_async_smem();
    tc_fence_before(); __syncthreads(); tc_fence_after();
    uint8_t *A = smem, *B = smem + 128 * 1024;
    const int rows = 632;
    const uint32_t LBO_A = rows * 16, LBO_B = N * 16;
    constexpr uint32_t ID = idesc_bf16_f32(128, N);
    unsigned long long t0 = clock64();
    const int wid = __shfl_sync(0xffffffff, (int)threadIdx.x / 32, 0);
    __shared__ volatile int stop;
    if (threadIdx.x == 0) stop = 0;
    __syncthreads();
    if ((MODE == 12 || MODE == 14) && wid >= 1) {
        // epilogue-like interference: tcgen05.ld of TMEM columns 384..511 (not used by the MMAs) in a loop
        const uint32_t tb = __shfl_sync(0xffffffff, tbase, 0);
        uint32_t r[16], acc = 0;
        while (!stop) {
            for (int c = 0; c < 128; c += 16) {
                tmem_ld16(tb + ((uint32_t)(wid * 32) << 16) + 384 + c, r);
                tmem_ld_wait();
                acc += r[0];
            }
        }
        if (acc == 12345) cyc[blockIdx.x + 1000] = acc;
    } else if ((MODE == 13 || MODE == 14) && wid == 1) {
        // loader-like interference: bulk copies of 32 KB into shared memory (region 160-192 KB, not read by the MMAs)
        uint32_t ph = 0;
        while (!stop) {
            if (elect_one()) {
                mbar_arrive_expect_tx(&wfull[0], 32768);
                bulk_g2s(smem + 160 * 1024, gw, 32768, &wfull[0]);
            }
            __syncwarp();
            mbar_wait(&wfull[0], ph);
            ph ^= 1;
        }
    }
    if (wid == 0) {
        const uint32_t tb = __shfl_sync(0xffffffff, tbase, 0);
        const uint32_t abase = smem_u32(A) >> 4, bbase = smem_u32(B) >> 4;
        if (MODE >= 11) {
            // depth-stacked cfg5 pattern: per k-step (18) six input planes, MMAs of N = 32, 64, 96, 96, 64, 32
            // (Td = 4), SW64 A (plane = 162 rows), B stacked [2][96][8] per k-step
            const uint64_t a0 = umma_desc_sw64(0, 512), b0 = umma_desc_noswz(0, 96 * 16, 128);
            const uint32_t nn[6] = {32, 64, 96, 96, 64, 32};
            const uint32_t bo[6] = {0, 0, 0, 0, 32, 64};
            const uint32_t col[6] = {96, 64, 32, 0, 0, 0};
            for (int it = 0; it < iters; it++) {
                for (int q = 0; q < 18; q++) {
                    const uint32_t px = ((q / 2) / 3) * 18 + (q / 2) % 3;
                    const uint64_t bd0 = b0 + bbase + q * (96 * 2);
#pragma unroll
                    for (int i = 0; i < 6; i++) {
                        const uint64_t ad = a0 + abase + (px + i * 162) * 4 + (q % 2) * 2;
                        mma_bf16_elect(tb + (it & 1) * 128 + col[i], ad, bd0 + bo[i], idesc_bf16_f32(128, nn[i]), 1);
                    }
                }
            }
        } else if (MODE == 9 || MODE == 10) {
            // generic-kernel cfg5 shape on the 64-B swizzled layout (AM_SW64): pixel rows of 64 B, Wp = 18, plane 288
            // rows, 27 taps x 2 k-steps, ntl = 2 (mode 9) or 1 (mode 10)
            const uint64_t a0 = umma_desc_sw64(0, 512), b0 = umma_desc_noswz(0, N * 16, 128);
            const int ntl = MODE == 9 ? 2 : 1;
            for (int it = 0; it < iters; it++) {
                for (int tap = 0; tap < 27; tap++) {
                    const uint32_t px = (tap / 9) * 288 + ((tap / 3) % 3) * 18 + tap % 3;
#pragma unroll
                    for (int kk = 0; kk < 2; kk++) {
                        uint64_t bd = b0 | ((bbase + (tap * 2 + kk) * (N * 2)) & 0x3FFF);
                        for (int tl = 0; tl < ntl; tl++) {
                            uint64_t ad = a0 | ((abase + (px + tl * 128) * 4 + kk * 2) & 0x3FFF);
                            mma_bf16_elect(tb + (it & 1) * 128 + tl * N, ad, bd, ID, 1);
                        }
                    }
                }
            }
        } else if (MODE == 7 || MODE == 8) {
            // generic-kernel cfg5 shape: chunk planes of 497 (7) or 496 (8) rows, 27 taps x 2 k-steps, ntl = 1
            const uint32_t rowsP = MODE == 7 ? 497 : 496;
            const uint32_t LBO7 = rowsP * 16;
            const uint64_t a0 = umma_desc_noswz(0, LBO7, 128), b0 = umma_desc_noswz(0, N * 16, 128);
            for (int it = 0; it < iters; it++) {
                for (int tap = 0; tap < 27; tap++) {
                    const uint32_t shift = (tap / 9) * 162 + ((tap / 3) % 3) * 18 + tap % 3;
#pragma unroll
                    for (int kk = 0; kk < 2; kk++) {
                        uint64_t ad = a0 | ((abase + shift + kk * 2 * (LBO7 >> 4)) & 0x3FFF);
                        uint64_t bd = b0 | ((bbase + (tap * 2 + kk) * (N * 2)) & 0x3FFF);
                        mma_bf16_elect(tb + (it & 1) * 64, ad, bd, ID, 1);
                    }
                }
            }
        } else if (MODE == 0) {
            const uint64_t a0 = umma_desc_noswz(0, LBO_A, 128), b0 = umma_desc_noswz(0, LBO_B, 128);
            for (int it = 0; it < iters; it++) {
#pragma unroll
                for (int k = 0; k < 16; k++) {
                    uint64_t ad = a0 | ((abase + (k % 4) * 2 * (LBO_A >> 4) + k * 7) & 0x3FFF);
                    uint64_t bd = b0 | ((bbase + (k % 4) * 2 * (LBO_B >> 4)) & 0x3FFF);
                    mma_bf16_elect(tb + (k & 1) * (N <= 128 ? 256 : 0), ad, bd, ID, 1);
                }
            }
        } else {
            const uint64_t a0 = umma_desc_sw128(0, 1024), b0 = umma_desc_noswz(0, LBO_B, 128);
            uint32_t wi = 0;
            const uint32_t WB = N * 64 * 2;
            for (int it = 0; it < iters; it++) {   // one "tap" per iteration: 4 tiles x 4 k-steps
                const uint32_t g = it;
                uint32_t bb = bbase;
                if (MODE == 3) {
                    mbar_wait(&wfull[g % 4], (g / 4) & 1);
                    tc_fence_after();
                    bb = (smem_u32(B) + (g % 4) * (N * 64 * 2)) >> 4;
                }
                if (MODE == 2) {
                    while (wi < g + 4 && (wi < 4 || g == 0)) {
                        const int st = wi % 4;
                        if (wi >= 4) mbar_wait(&wempty[st], ((wi / 4) - 1) & 1);
                        if (elect_one()) {
                            mbar_arrive_expect_tx(&wfull[st], WB);
                            bulk_g2s(B + st * WB, gw + (size_t)(wi % 9) * WB, WB, &wfull[st]);
                        }
                        __syncwarp();
                        wi++;
                    }
                    mbar_wait(&wfull[g % 4], (g / 4) & 1);
                    tc_fence_after();
                    bb = (smem_u32(B) + (g % 4) * WB) >> 4;
                }
                uint32_t shift = (it % 9) / 3 * 58 + (it % 3);
                if (MODE == 5) shift = shift / 8 * 8;        // 1024-B aligned A starts
                if (MODE == 6) shift = 0;                    // same A every tap
#pragma unroll
                for (int t = 0; t < (MODE >= 4 ? 3 : 4); t++)
#pragma unroll
                    for (int kk = 0; kk < 4; kk++) {
                        uint64_t ad = a0 | ((abase + (shift + t * 128) * 8 + kk * 2) & 0x3FFF);
                        uint64_t bd = b0 | ((bb + kk * 2 * (LBO_B >> 4)) & 0x3FFF);
                        mma_bf16_elect(tb + (N > 128 ? 0 : t * N), ad, bd, ID, 1);
                    }
                if (MODE == 3) mma_commit_elect(&wempty[g % 4]);
                if (MODE == 2) {
                    mma_commit_elect(&wempty[g % 4]);
                    while (wi < g + 4) {   // refill the stage of tap g-1 while tap g's MMAs run
                        const int st = wi % 4;
                        if (wi >= 4) mbar_wait(&wempty[st], ((wi / 4) - 1) & 1);
                        if (elect_one()) {
                            mbar_arrive_expect_tx(&wfull[st], WB);
                            bulk_g2s(B + st * WB, gw + (size_t)(wi % 9) * WB, WB, &wfull[st]);
                        }
                        __syncwarp();
                        wi++;
                    }
                }
            }
        }
        mma_commit_elect(&done);
    } else if (MODE == 3 && wid == 1) {
        const uint32_t WB = N * 64 * 2;
        for (uint32_t wi = 0; wi < (uint32_t)iters; wi++) {
            const int st = wi % 4;
            if (wi >= 4) mbar_wait(&wempty[st], ((wi / 4) - 1) & 1);
            if (elect_one()) {
                mbar_arrive_expect_tx(&wfull[st], WB);
                bulk_g2s(B + st * WB, gw + (size_t)(wi % 9) * WB, WB, &wfull[st]);
            }
            __syncwarp();
        }
    }
    if (wid == 0) {
        mbar_wait(&done, 0);
        if (threadIdx.x == 0) stop = 1;
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    tc_fence_before(); __syncthreads();
    if (threadIdx.x < 32) tmem_dealloc(tbase, 512);
}

template <int N, int MODE> void run(int sms, const uint8_t *gw) {
    unsigned long long *d; cudaMalloc(&d, sms * 8);
    int iters = 2000;
    cudaFuncSetAttribute(mma_loop<N, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    mma_loop<N, MODE><<<sms, 128, 200 * 1024>>>(10, d, gw);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    mma_loop<N, MODE><<<sms, 128, 200 * 1024>>>(iters, d, gw);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    unsigned long long h[256]; cudaMemcpy(h, d, sms * 8, cudaMemcpyDeviceToHost);
    double n_mma = (double)iters * (MODE >= 11 ? 108 : MODE == 9 ? 108 : MODE >= 7 ? 54 : MODE >= 4 ? 12 : 16);
    double flops = n_mma * 2.0 * 128 * N * 16 * sms;
    printf("mode=%d N=%3d  cycles/MMA=%.1f (ideal %d)  chip %.1f TFLOP/s  (%s)\n", MODE, N, h[0] / n_mma, 128 * N / 256,
           flops / (ms * 1e-3) / 1e12, cudaGetErrorString(cudaGetLastError()));
    fflush(stdout);
    cudaFree(d);
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint8_t *gw; cudaMalloc(&gw, 9 * 64 * 64 * 2 * 4); cudaMemset(gw, 0, 9 * 64 * 64 * 2 * 4);
    run<32, 0>(sms, gw); run<64, 0>(sms, gw); run<128, 0>(sms, gw); run<256, 0>(sms, gw);
    run<64, 1>(sms, gw); run<64, 2>(sms, gw); run<64, 3>(sms, gw);
    run<64, 4>(sms, gw); run<64, 5>(sms, gw); run<64, 6>(sms, gw);
    run<64, 4>(1, gw); run<64, 5>(1, gw); run<64, 6>(1, gw);
    run<192, 0>(sms, gw); run<192, 4>(sms, gw); run<128, 4>(sms, gw); run<256, 4>(sms, gw);
    run<32, 7>(sms, gw); run<32, 8>(sms, gw); run<32, 0>(sms, gw);
    run<32, 9>(sms, gw); run<32, 10>(sms, gw); run<32, 11>(sms, gw); run<32, 12>(sms, gw); run<32, 13>(sms, gw);
    run<32, 14>(sms, gw);
    return 0;
}
