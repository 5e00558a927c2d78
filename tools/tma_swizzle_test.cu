// Does a TMA tiled load with SWIZZLE_128B into a shared-memory destination that is 128-B but not
// 1024-B aligned apply the swizzle by absolute address bits (chunk ^= addr bits [7:9])?
#include <cstdio>
#include <cstdint>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include "../paper_conf_icpp_lakshminarasimhan24_b200/csrc/kernels/tc_ptx.cuh"
using namespace bdl::ptx;

__global__ void k(const __grid_constant__ CUtensorMap tm, int q, int row0, int *bad) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    for (int i = threadIdx.x; i < 32 * 1024 / 16; i += blockDim.x) *(uint4 *)(smem + i * 16) = make_uint4(0xffffffff, 0, 0, 0);
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    fence_proxy_async_smem();
    __syncthreads();
    uint8_t *dst = smem + 1024 + q * 128;
    if (threadIdx.x == 0) {
        mbar_arrive_expect_tx(&bar, 1024);
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                     :: "r"(smem_u32(dst)), "l"(&tm), "r"(0), "r"(row0), "r"(smem_u32(&bar)) : "memory");
    }
    mbar_wait(&bar, 0);
    // verify: element (i, c*8 + e) of the box; value encodes row*64 + col
    int errs = 0;
    for (int i = 0; i < 8; i++) for (int c = 0; c < 8; c++) {
        uint32_t addr = smem_u32(dst) + i * 128;
        int sc = c ^ ((addr >> 7) & 7);
        const __nv_bfloat16 *p = (const __nv_bfloat16 *)(dst + i * 128 + sc * 16);
        for (int e = 0; e < 8; e++) {
            float want = (float)(((row0 + i) * 64 + c * 8 + e) % 251);
            if (__bfloat162float(p[e]) != want) errs++;
        }
    }
    if (threadIdx.x == 0) *bad = errs;
}

int main() {
    const int R = 4096;
    __nv_bfloat16 *h = new __nv_bfloat16[R * 64];
    for (int i = 0; i < R * 64; i++) h[i] = __float2bfloat16((float)(i % 251));
    __nv_bfloat16 *d; cudaMalloc(&d, R * 64 * 2); cudaMemcpy(d, h, R * 64 * 2, cudaMemcpyHostToDevice);
    PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    cudaDriverEntryPointQueryResult qr;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &qr);
    if (!enc) { printf("no entry point\n"); return 1; }
    CUtensorMap tm;
    cuuint64_t dims[2] = {64, (cuuint64_t)R};
    cuuint64_t strides[1] = {128};
    cuuint32_t box[2] = {64, 8};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode %d\n", (int)r);
    int *bad; cudaMalloc(&bad, 4);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 40 * 1024);
    for (int q = 0; q < 10; q++) {
        k<<<1, 128, 40 * 1024>>>(tm, q, 17 + q, bad);
        cudaError_t e = cudaDeviceSynchronize();
        int hb = -1; cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
        printf("dst offset %d x 128 B: %s, mismatches %d\n", q, cudaGetErrorString(e), hb);
    }
    return 0;
}
