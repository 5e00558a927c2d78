// CTA-pair tcgen05 probe (B200): (1) layout of a cta_group::2 kind::f16 MMA with M = 256, N = 64 -- which CTA's
// shared memory holds which half of B, where each CTA's D rows land -- checked element by element against a host
// product; (2) cycles per MMA of the cfg2 band pattern (3 M tiles x 9 shifted taps x 4 k-steps, weights resident)
// for the pair (M = 256, half of B per CTA) against one CTA (M = 128, all of B).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/pair_mma_test.cu -o tools/pair_mma_test
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <vector>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include "../paper_conf_icpp_lakshminarasimhan24_b200/csrc/kernels/tc_ptx.cuh"
using namespace bdl::ptx;

// A: 128 rows x 64 k bf16, 128-B swizzled rows; B: 32 (pair) or 64 (single) rows x 64 k, [8 k-chunks][rows][8]
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1)
    pair_layout(const __nv_bfloat16 *gA, const __nv_bfloat16 *gB, float *out) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t done;
    __shared__ uint32_t tbase;
    const uint32_t rank = cluster_rank();
    uint8_t *A = smem, *B = smem + 16384;
    for (int i = threadIdx.x; i < 128 * 8; i += 128) {
        const int m = i / 8, j = i % 8;
        *(uint4 *)(A + m * 128 + ((j ^ (m & 7)) * 16)) = *(const uint4 *)(gA + ((size_t)rank * 128 + m) * 64 + j * 8);
    }
    for (int i = threadIdx.x; i < 32 * 8; i += 128) {
        const int n = i / 8, j = i % 8;
        *(uint4 *)(B + j * 512 + n * 16) = *(const uint4 *)(gB + ((size_t)rank * 32 + n) * 64 + j * 8);
    }
    if (threadIdx.x == 0) {
        mbar_init(&done, 1);
        fence_barrier_init();
    }
    if (threadIdx.x < 32) tmem_alloc2(&tbase, 64);
    fence_proxy_async_smem();
    tc_fence_before();
    cluster_sync();
    tc_fence_after();
    const uint32_t tb = tbase;
    if (rank == 0 && threadIdx.x < 32) {
        const uint64_t a0 = umma_desc_sw128(smem_u32(A), 1024), b0 = umma_desc_noswz(smem_u32(B), 512, 128);
        for (int kk = 0; kk < 4; kk++) mma2_bf16_elect(tb, a0 + kk * 2, b0 + kk * 64, idesc_bf16_f32(256, 64), kk > 0);
        mma2_commit_mc(&done, 3);
    }
    mbar_wait(&done, 0);
    tc_fence_after();
    const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
    uint32_t r[16];
    for (int c = 0; c < 64; c += 16) {
        tmem_ld16(tb + ((uint32_t)(w * 32) << 16) + c, r);
        tmem_ld_wait();
        for (int e = 0; e < 16; e++) out[((size_t)rank * 128 + w * 32 + lane) * 64 + c + e] = __uint_as_float(r[e]);
    }
    tc_fence_before();
    cluster_sync();
    if (threadIdx.x < 32) {
        tmem_relinquish2();
        tmem_dealloc2(tb, 64);
    }
}

// Throughput: PAIR = 1: leader issues M = 256 MMAs (B rows 32 per CTA); PAIR = 0: every CTA issues M = 128 (B rows 64).
// LOAD = 1: a second warp streams 59 KB per task into a separate buffer by bulk copies (the input-tile TMA writes).
template <int PAIR, int LOAD>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1)
    band_tput(int tasks, unsigned long long *cyc, const uint8_t *gsrc) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t done, lfull;
    __shared__ uint32_t tbase;
    __shared__ volatile int stop;
    const uint32_t rank = cluster_rank();
    constexpr int NB = PAIR ? 32 : 64;
    uint8_t *A = smem, *Wt = smem + 504 * 128, *L = Wt + 9 * NB * 128;
    for (int i = threadIdx.x * 16; i < 504 * 128 + 9 * NB * 128; i += 128 * 16) *(uint4 *)(smem + i) = make_uint4(0, 0, 0, 0);
    if (threadIdx.x == 0) {
        mbar_init(&done, 1);
        mbar_init(&lfull, 1);
        stop = 0;
        fence_barrier_init();
    }
    if (threadIdx.x < 32) {
        if (PAIR) tmem_alloc2(&tbase, 512);
        else tmem_alloc(&tbase, 512);
    }
    fence_proxy_async_smem();
    tc_fence_before();
    cluster_sync();
    tc_fence_after();
    const uint32_t tb = tbase;
    const int w = threadIdx.x / 32;
    unsigned long long t0 = clock64();
    if (w == 0 && (!PAIR || rank == 0)) {
        const uint64_t a0 = umma_desc_sw128(smem_u32(A), 1024), b0 = umma_desc_noswz(smem_u32(Wt), NB * 16, 128);
        constexpr uint32_t ID = idesc_bf16_f32(PAIR ? 256 : 128, 64);
        for (int t = 0; t < tasks; t++) {
            const uint32_t d = tb + (t & 1) * 192;
            for (int tap = 0; tap < 9; tap++) {
                const uint32_t shift = (tap / 3) * 58 + tap % 3;
#pragma unroll
                for (int tl = 0; tl < 3; tl++)
#pragma unroll
                    for (int kk = 0; kk < 4; kk++) {
                        const uint64_t ad = a0 + (shift + tl * 128) * 8 + kk * 2;
                        const uint64_t bd = b0 + tap * (NB * 8) + kk * (NB * 2);
                        if (PAIR) mma2_bf16_elect(d + tl * 64, ad, bd, ID, (tap | kk) != 0);
                        else mma_bf16_elect_nc(d + tl * 64, ad, bd, ID, (tap | kk) != 0);
                    }
            }
        }
        if (PAIR) mma2_commit_mc(&done, 3);
        else mma_commit_elect(&done);
    } else if (LOAD && w == 1) {
        uint32_t ph = 0;
        while (!stop) {
            if (elect_one()) {
                mbar_arrive_expect_tx(&lfull, 59 * 1024);
                bulk_g2s(L, gsrc, 59 * 1024, &lfull);
            }
            __syncwarp();
            mbar_wait(&lfull, ph);
            ph ^= 1;
            // one tile load per ~108 MMAs at ~40 cycles
            const unsigned long long s = clock64();
            while (clock64() - s < 4000) {}
        }
    }
    if (w == 0) {
        mbar_wait(&done, 0);
        if (threadIdx.x == 0) stop = 1;
    }
    __syncthreads();
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    tc_fence_before();
    cluster_sync();
    if (threadIdx.x < 32) {
        if (PAIR) {
            tmem_relinquish2();
            tmem_dealloc2(tb, 512);
        } else {
            tmem_relinquish();
            tmem_dealloc(tb, 512);
        }
    }
}

template <int PAIR, int LOAD>
void tput(int sms, const uint8_t *src) {
    unsigned long long *d;
    cudaMalloc(&d, sms * 8);
    const int smem = 504 * 128 + 9 * (PAIR ? 32 : 64) * 128 + 60 * 1024;
    cudaFuncSetAttribute(band_tput<PAIR, LOAD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    band_tput<PAIR, LOAD><<<sms, 128, smem>>>(4, d, src);
    const int tasks = 400;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    band_tput<PAIR, LOAD><<<sms, 128, smem>>>(tasks, d, src);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    std::vector<unsigned long long> h(sms);
    cudaMemcpy(h.data(), d, sms * 8, cudaMemcpyDeviceToHost);
    const double mma_per_sm = tasks * 108.0;   // M = 128 x N = 64 x K = 16 units per SM
    const double flops = mma_per_sm * 2.0 * 128 * 64 * 16 * sms;
    printf("%s%s: cycles per 128x64x16 per SM = %.1f (ideal 32)  chip %.0f TFLOP/s  (%s)\n", PAIR ? "pair M=256" : "single M=128",
           LOAD ? " + 59 KB bulk load per task" : "", h[0] / mma_per_sm, flops / (ms * 1e-3) / 1e12,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(d);
}

int main() {
    // (1) layout
    std::vector<__nv_bfloat16> hA(256 * 64), hB(64 * 64);
    std::vector<float> fA(256 * 64), fB(64 * 64);
    for (int m = 0; m < 256; m++)
        for (int k = 0; k < 64; k++) {
            float v = (float)((m * 3 + k * 5 + (m / 128) * 7) % 7 - 3);
            hA[m * 64 + k] = __float2bfloat16(v);
            fA[m * 64 + k] = v;
        }
    for (int n = 0; n < 64; n++)
        for (int k = 0; k < 64; k++) {
            float v = (float)((n * 11 + k * 2 + n / 32 * 13) % 5 - 2);
            hB[n * 64 + k] = __float2bfloat16(v);
            fB[n * 64 + k] = v;
        }
    __nv_bfloat16 *dA, *dB;
    float *dO;
    cudaMalloc(&dA, hA.size() * 2);
    cudaMalloc(&dB, hB.size() * 2);
    cudaMalloc(&dO, 256 * 64 * 4);
    cudaMemcpy(dA, hA.data(), hA.size() * 2, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB.data(), hB.size() * 2, cudaMemcpyHostToDevice);
    cudaMemset(dO, 0, 256 * 64 * 4);
    cudaFuncSetAttribute(pair_layout, cudaFuncAttributeMaxDynamicSharedMemorySize, 32768);
    pair_layout<<<2, 128, 32768>>>(dA, dB, dO);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<float> o(256 * 64);
    cudaMemcpy(o.data(), dO, o.size() * 4, cudaMemcpyDeviceToHost);
    // hypothesis: D row m (CTA m / 128) col n = sum_k A[m][k] * B[n][k], B rows 0..31 from the leader, 32..63 from the peer
    double err = 0;
    for (int m = 0; m < 256; m++)
        for (int n = 0; n < 64; n++) {
            double s = 0;
            for (int k = 0; k < 64; k++) s += (double)fA[m * 64 + k] * fB[n * 64 + k];
            err = std::max(err, std::abs(s - o[m * 64 + n]));
        }
    printf("pair layout (%s): max |D - A B^T| = %g  (0 => leader holds B columns 0..N/2-1, CTA r holds D rows 128r..)\n",
           cudaGetErrorString(e), err);
    if (err != 0) {
        printf("sample D[0][0..3] %g %g %g %g, D[128][0..3] %g %g %g %g\n", o[0], o[1], o[2], o[3], o[128 * 64], o[128 * 64 + 1],
               o[128 * 64 + 2], o[128 * 64 + 3]);
    }
    // (2) throughput
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint8_t *src;
    cudaMalloc(&src, 64 * 1024);
    cudaMemset(src, 0, 64 * 1024);
    tput<0, 0>(sms, src);
    tput<1, 0>(sms, src);
    tput<0, 1>(sms, src);
    tput<1, 1>(sms, src);
    return err == 0 ? 0 : 1;
}
