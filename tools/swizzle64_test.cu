// Does a K-major SWIZZLE_64B UMMA A-operand (pixel rows of 64 B = 32 bf16 channels) tolerate a start
// address shifted by whole 64-B rows, like SWIZZLE_128B does (tools/swizzle_test.cu)?  A = 256 rows x 32
// bf16, written with the absolute-address 64-B swizzle (16-B chunk ^= addr bits [7:8]); B = 32 x 32 bf16
// (no swizzle, chunk-major).  For shift s: D[m][n] = sum_k A[s+m][k] * B[n][k] (M=128, N=32, K=32).
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_bf16.h>
#include "../paper_conf_icpp_lakshminarasimhan24_b200/csrc/kernels/tc_ptx.cuh"
using namespace bdl::ptx;

__global__ void k(const __nv_bfloat16 *A, const __nv_bfloat16 *B, float *D, int shift) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tb;
    uint8_t *As = smem, *Bs = smem + 64 * 1024;
    for (int i = threadIdx.x; i < 256 * 4; i += blockDim.x) {
        int r = i / 4, c = i % 4;
        uint32_t row_addr = smem_u32(As) + r * 64;
        int sc = c ^ ((row_addr >> 7) & 3);
        *(uint4 *)(As + r * 64 + sc * 16) = *(const uint4 *)(A + r * 32 + c * 8);
    }
    for (int i = threadIdx.x; i < 32 * 4; i += blockDim.x) {
        int n = i / 4, c = i % 4;
        *(uint4 *)(Bs + (c * 32 + n) * 16) = *(const uint4 *)(B + n * 32 + c * 8);
    }
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    if (threadIdx.x < 32) { tmem_alloc(&tb, 32); tmem_relinquish(); }
    fence_proxy_async_smem();
    tc_fence_before(); __syncthreads(); tc_fence_after();
    if (threadIdx.x < 32) {
        const uint32_t idesc = idesc_bf16_f32(128, 32);
        for (int kk = 0; kk < 2; kk++) {
            uint32_t a_addr = smem_u32(As) + shift * 64 + kk * 32;
            uint64_t ad = 0;
            ad |= (uint64_t)((a_addr >> 4) & 0x3FFF);
            ad |= (uint64_t)(1) << 16;
            ad |= (uint64_t)((512 >> 4) & 0x3FFF) << 32;   // SBO = 8 rows x 64 B
            ad |= (uint64_t)1 << 46;
            ad |= (uint64_t)4 << 61;                        // SWIZZLE_64B
            uint64_t bd = umma_desc_noswz(smem_u32(Bs) + kk * 2 * 512, 512, 128);
            mma_bf16_elect(tb, ad, bd, idesc, kk > 0);
        }
        mma_commit_elect(&bar);
    }
    mbar_wait(&bar, 0);
    tc_fence_after();
    uint32_t r[16];
    for (int c = 0; c < 2; c++) {
        tmem_ld16(tb + ((threadIdx.x / 32 * 32) << 16) + c * 16, r);
        tmem_ld_wait();
        reg_fence16(r);
        for (int e = 0; e < 16; e++) D[threadIdx.x * 32 + c * 16 + e] = __uint_as_float(r[e]);
    }
    tc_fence_before(); __syncthreads();
    if (threadIdx.x < 32) tmem_dealloc(tb, 32);
}

int main() {
    const int NA = 256 * 32, NB = 32 * 32;
    __nv_bfloat16 *hA = new __nv_bfloat16[NA], *hB = new __nv_bfloat16[NB];
    float *fA = new float[NA], *fB = new float[NB];
    for (int i = 0; i < NA; i++) { float v = (float)((i * 37 % 101) - 50) / 32.f; hA[i] = __float2bfloat16(v); fA[i] = __bfloat162float(hA[i]); }
    for (int i = 0; i < NB; i++) { float v = (float)((i * 53 % 97) - 48) / 64.f; hB[i] = __float2bfloat16(v); fB[i] = __bfloat162float(hB[i]); }
    __nv_bfloat16 *dA, *dB; float *dD;
    cudaMalloc(&dA, NA * 2); cudaMalloc(&dB, NB * 2); cudaMalloc(&dD, 128 * 32 * 4);
    cudaMemcpy(dA, hA, NA * 2, cudaMemcpyHostToDevice); cudaMemcpy(dB, hB, NB * 2, cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    float *hD = new float[128 * 32];
    int ok = 0;
    for (int s = 0; s < 12; s++) {
        k<<<1, 128, 100 * 1024>>>(dA, dB, dD, s);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
        cudaMemcpy(hD, dD, 128 * 32 * 4, cudaMemcpyDeviceToHost);
        double maxerr = 0;
        for (int m = 0; m < 128; m++) for (int n = 0; n < 32; n++) {
            double ref = 0; for (int kq = 0; kq < 32; kq++) ref += (double)fA[(s + m) * 32 + kq] * fB[n * 32 + kq];
            maxerr = fmax(maxerr, fabs(ref - hD[m * 32 + n]));
        }
        printf("swizzle64 shift=%d maxerr=%g\n", s, maxerr);
        ok += maxerr < 1e-2;
    }
    printf("=> %d/12 shifts correct\n", ok);
    return 0;
}
