// Does a K-major SWIZZLE_128B UMMA A-operand tolerate a start address shifted by whole 128-B rows
// (i.e. not 1024-B aligned)?  A = 256 pixel rows x 64 bf16 (128 B), written with the absolute-address
// 128-B swizzle (chunk ^= addr bits [7:9]); B = 64 x 64 bf16 (no swizzle).  For shift s the MMA must
// produce D[m][n] = sum_k A[s+m][k] * B[n][k].  Tries base_offset = 0 and = (s & 7).
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_bf16.h>
#include "../paper_conf_icpp_lakshminarasimhan24_b200/csrc/kernels/tc_ptx.cuh"
using namespace bdl::ptx;

__global__ void k(const __nv_bfloat16 *A, const __nv_bfloat16 *B, float *D, int shift, int use_bo, int swz_mode) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tb;
    uint8_t *As = smem, *Bs = smem + 64 * 1024;
    // A: 256 rows x 128 B, swizzled by absolute address bits
    for (int i = threadIdx.x; i < 256 * 8; i += blockDim.x) {
        int r = i / 8, c = i % 8;
        uint32_t row_addr = smem_u32(As) + r * 128;
        int sc = swz_mode ? (c ^ ((row_addr >> 7) & 7)) : c;
        *(uint4 *)(As + r * 128 + sc * 16) = *(const uint4 *)(A + r * 64 + c * 8);
    }
    // B: no swizzle, chunk-major [8][64 rows][16 B]
    for (int i = threadIdx.x; i < 64 * 8; i += blockDim.x) {
        int n = i / 8, c = i % 8;
        *(uint4 *)(Bs + (c * 64 + n) * 16) = *(const uint4 *)(B + n * 64 + c * 8);
    }
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    if (threadIdx.x < 32) { tmem_alloc(&tb, 64); tmem_relinquish(); }
    fence_proxy_async_smem();
    tc_fence_before(); __syncthreads(); tc_fence_after();
    if (threadIdx.x < 32) {
        const uint32_t idesc = idesc_bf16_f32(128, 64);
        for (int kk = 0; kk < 4; kk++) {
            uint32_t a_addr = smem_u32(As) + shift * 128 + kk * 32;
            uint64_t ad = 0;
            ad |= (uint64_t)((a_addr >> 4) & 0x3FFF);
            ad |= (uint64_t)(1) << 16;                 // LBO (unused for swizzled K-major)
            ad |= (uint64_t)((1024 >> 4) & 0x3FFF) << 32;  // SBO = 8 rows x 128 B
            ad |= (uint64_t)1 << 46;
            if (use_bo) ad |= (uint64_t)((a_addr >> 7) & 7) << 49;
            ad |= (uint64_t)2 << 61;                   // SWIZZLE_128B
            uint64_t bd = umma_desc_noswz(smem_u32(Bs) + kk * 2 * 1024, 1024, 128);
            mma_bf16_elect(tb, ad, bd, idesc, kk > 0);
        }
        mma_commit_elect(&bar);
    }
    mbar_wait(&bar, 0);
    tc_fence_after();
    uint32_t r[16];
    for (int c = 0; c < 4; c++) {
        tmem_ld16(tb + ((threadIdx.x / 32 * 32) << 16) + c * 16, r);
        tmem_ld_wait();
        reg_fence16(r);
        for (int e = 0; e < 16; e++) D[threadIdx.x * 64 + c * 16 + e] = __uint_as_float(r[e]);
    }
    tc_fence_before(); __syncthreads();
    if (threadIdx.x < 32) tmem_dealloc(tb, 64);
}

int main() {
    const int NA = 256 * 64, NB = 64 * 64;
    __nv_bfloat16 *hA = new __nv_bfloat16[NA], *hB = new __nv_bfloat16[NB];
    float *fA = new float[NA], *fB = new float[NB];
    for (int i = 0; i < NA; i++) { float v = (float)((i * 37 % 101) - 50) / 32.f; hA[i] = __float2bfloat16(v); fA[i] = __bfloat162float(hA[i]); }
    for (int i = 0; i < NB; i++) { float v = (float)((i * 53 % 97) - 48) / 64.f; hB[i] = __float2bfloat16(v); fB[i] = __bfloat162float(hB[i]); }
    __nv_bfloat16 *dA, *dB; float *dD;
    cudaMalloc(&dA, NA * 2); cudaMalloc(&dB, NB * 2); cudaMalloc(&dD, 128 * 64 * 4);
    cudaMemcpy(dA, hA, NA * 2, cudaMemcpyHostToDevice); cudaMemcpy(dB, hB, NB * 2, cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
    float *hD = new float[128 * 64];
    for (int use_bo = 0; use_bo < 2; use_bo++) {
        int ok_shifts = 0;
        for (int s = 0; s < 10; s++) {
            k<<<1, 128, 100 * 1024>>>(dA, dB, dD, s, use_bo, 1);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
            cudaMemcpy(hD, dD, 128 * 64 * 4, cudaMemcpyDeviceToHost);
            double maxerr = 0;
            for (int m = 0; m < 128; m++) for (int n = 0; n < 64; n++) {
                double ref = 0; for (int kq = 0; kq < 64; kq++) ref += (double)fA[(s + m) * 64 + kq] * fB[n * 64 + kq];
                maxerr = fmax(maxerr, fabs(ref - hD[m * 64 + n]));
            }
            printf("swizzle128 base_offset=%s shift=%d maxerr=%g\n", use_bo ? "addr" : "0", s, maxerr);
            ok_shifts += maxerr < 1e-2;
        }
        printf("=> base_offset=%s: %d/10 shifts correct\n", use_bo ? "addr" : "0", ok_shifts);
    }
    return 0;
}
