// TMA-staged brickify / unbrickify for 2-D bf16 tensors with C % 64 == 0 (the tcgen05 configs).
//
// One CTA converts R image rows x all W pixels x 64 channels of one sample:
//   brickify:   TMA load of the NCHW box (64 px, 64 ch, R rows) through a 5-D view that splits the
//               channel c = 8g + k so the box lands as smem [xb][row][k][g][128 B] (128-B swizzled);
//               a thread owns 8 channels (group g) x 8 pixels: for each k the 8 lanes of a group read 8
//               consecutive swizzled rows (conflict-free), transpose 8x8 in registers, and store the 8
//               pixel chunks g straight to the bricked tensor (the 8 lanes of a group fill one pixel's 128 B).
//   unbrickify: the reverse (TMA row load of bricks, transpose, TMA store of NCHW boxes).
// Dense-side traffic moves through the TMA engine; shared-memory accesses are 16-byte and conflict-free.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <string>

#include "common.cuh"
#include "tc_ptx.cuh"

namespace bdl {

struct TmaConvParams {
    CUtensorMap dense;    // NCHW as (W, C/8, 8, H, N) [c = 8g + k]: box (64 px, 8, 8, R rows, 1)
    CUtensorMap bricks;   // bricked (ch, xin, bx, yin, brick-row): box (64 ch, Bw, nbx, 1, 1)
    int N, C, H, W;
    int R;                // image rows per CTA
    int Bh, Bw, lBh, lBw;
    int nbx, nbh;         // bricks along w, h
    int nxb;              // 64-pixel boxes along w
    int ncb;              // 64-channel blocks
    void *out;            // brickify: the bricked tensor (direct stores)
    int Cp;               // padded channels
    long long brick_elems;
};

// 128-B swizzle: 16-B chunk j of the 128-B row at shared address `row` lives at chunk j ^ (row bits 7..9)
__device__ __forceinline__ uint8_t *swz(uint8_t *row, int j) {
    return row + ((j ^ ((ptx::smem_u32(row) >> 7) & 7)) << 4);
}

// 8x8 transpose of bf16: in[k] = 8 values of row k; out[i] = column i.
__device__ __forceinline__ void transpose8(const uint4 (&in)[8], uint4 (&out)[8]) {
    const uint16_t *e[8];
#pragma unroll
    for (int k = 0; k < 8; k++) e[k] = reinterpret_cast<const uint16_t *>(&in[k]);
#pragma unroll
    for (int i = 0; i < 8; i++) {
        uint32_t w0 = e[0][i] | ((uint32_t)e[1][i] << 16), w1 = e[2][i] | ((uint32_t)e[3][i] << 16);
        uint32_t w2 = e[4][i] | ((uint32_t)e[5][i] << 16), w3 = e[6][i] | ((uint32_t)e[7][i] << 16);
        out[i] = make_uint4(w0, w1, w2, w3);
    }
}

// smem: A = dense tile [nxb][R][64 ch][128 B].  The transposed 8-channel pixel chunks go straight to the bricked
// tensor: the 8 lanes of a group write the 8 chunks of one pixel (one 128-B line), so the stores are coalesced and no
// staging tile is needed -- 16 KB of shared memory per CTA (R = 2) lets the whole grid run in one wave.
__global__ void __launch_bounds__(128) brickify_tma_kernel(const __grid_constant__ TmaConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    pdl_launch_dependents();
    const int cb = blockIdx.x % p.ncb;
    const int rb = (blockIdx.x / p.ncb) % (p.nbh * p.Bh / p.R);
    const int n = blockIdx.x / p.ncb / (p.nbh * p.Bh / p.R);
    const int y0 = rb * p.R;
    const int Wg = p.nbx * p.Bw;
    uint8_t *A = smem;
    if (threadIdx.x == 0) {
        ptx::mbar_init(&bar, 1);
        ptx::fence_barrier_init();
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const uint32_t bytes = (uint32_t)p.nxb * p.R * 64 * 128;
        ptx::mbar_arrive_expect_tx(&bar, bytes);
        for (int xb = 0; xb < p.nxb; xb++)  // rows beyond H / columns beyond W / channels beyond C: zero fill
            ptx::tma_load_5d(A + (size_t)xb * p.R * 64 * 128, &p.dense, xb * 64, cb * 8, 0, y0, n, &bar);
    }
    ptx::mbar_wait(&bar, 0);
    // each item: one row, 8 channels (group g), 8 pixels (group q) -> 8 pixel chunks
    const int nq = Wg / 8;
    const int items = p.R * 8 * nq;
    uint8_t *out_base = reinterpret_cast<uint8_t *>(p.out);
    for (int it = threadIdx.x; it < items; it += blockDim.x) {
        const int g = it % 8;
        const int q = (it / 8) % nq;
        const int r = it / 8 / nq;
        const int y = y0 + r;
        if (y >= p.nbh * p.Bh) break;
        const int xb = q / 8, j = q % 8;
        uint4 in[8], out[8];
#pragma unroll
        for (int k = 0; k < 8; k++) {
            uint8_t *row = A + ((((size_t)xb * p.R + r) * 8 + k) * 8 + g) * 128;
            in[k] = *reinterpret_cast<const uint4 *>(swz(row, j));
        }
        transpose8(in, out);
        // pixels x = 8q .. 8q+7: one brick when Bw >= 8 (consecutive pixels Cp channels apart), else Bw-pixel runs
        const long long brow = ((long long)n * p.nbh + (y >> p.lBh)) * p.nbx;
        const int yin = (y & (p.Bh - 1)) << p.lBw;
        if (p.Bw >= 8) {
            const long long off = (brow + ((q * 8) >> p.lBw)) * p.brick_elems +
                                  (long long)(yin + ((q * 8) & (p.Bw - 1))) * p.Cp + cb * 64 + g * 8;
            uint4 *dst = reinterpret_cast<uint4 *>(out_base + off * 2);
            const int step = p.Cp / 8;   // 16-B vectors per pixel
#pragma unroll
            for (int i = 0; i < 8; i++) dst[i * step] = out[i];
        } else {
#pragma unroll
            for (int i = 0; i < 8; i++) {
                const int x = q * 8 + i;
                const long long off = (brow + (x >> p.lBw)) * p.brick_elems +
                                      (long long)(yin + (x & (p.Bw - 1))) * p.Cp + cb * 64 + g * 8;
                *reinterpret_cast<uint4 *>(out_base + off * 2) = out[i];
            }
        }
    }
}

__global__ void __launch_bounds__(128) unbrickify_tma_kernel(const __grid_constant__ TmaConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    const int cb = blockIdx.x % p.ncb;
    const int rb = (blockIdx.x / p.ncb) % ((p.H + p.R - 1) / p.R);
    const int n = blockIdx.x / p.ncb / ((p.H + p.R - 1) / p.R);
    const int y0 = rb * p.R;
    const int Wg = p.nbx * p.Bw;
    uint8_t *A = smem;                                        // dense tile [nxb][R][64][128 B]
    uint8_t *B = smem + (size_t)p.nxb * p.R * 64 * 128;       // brick rows [R][Wg][128 B]
    if (threadIdx.x == 0) {
        ptx::mbar_init(&bar, 1);
        ptx::fence_barrier_init();
    }
    __syncthreads();
    pdl_wait();  // launched with PDL after the subgraph kernel
    const int nr = min(p.R, p.H - y0);
    if (threadIdx.x == 0) {
        ptx::mbar_arrive_expect_tx(&bar, (uint32_t)nr * Wg * 128);
        for (int r = 0; r < nr; r++) {
            const int y = y0 + r;
            ptx::tma_load_5d(B + (size_t)r * Wg * 128, &p.bricks, cb * 64, 0, 0, y & (p.Bh - 1), n * p.nbh + (y >> p.lBh), &bar);
        }
    }
    ptx::mbar_wait(&bar, 0);
    const int nq = p.nxb * 8;   // 8-pixel groups of the dense tile (covers W, clipped by the store)
    const int items = nr * 8 * nq;
    for (int it = threadIdx.x; it < items; it += blockDim.x) {
        const int g = it % 8;
        const int q = (it / 8) % nq;
        const int r = it / 8 / nq;
        const int xb = q / 8, j = q % 8;
        uint4 in[8], out[8];
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const int x = q * 8 + i;
            in[i] = x < Wg ? *reinterpret_cast<const uint4 *>(swz(B + ((size_t)r * Wg + x) * 128, g)) : make_uint4(0, 0, 0, 0);
        }
        transpose8(in, out);
#pragma unroll
        for (int k = 0; k < 8; k++) {
            uint8_t *row = A + ((((size_t)xb * p.R + r) * 8 + k) * 8 + g) * 128;
            *reinterpret_cast<uint4 *>(swz(row, j)) = out[k];
        }
    }
    ptx::fence_proxy_async_smem();
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int xb = 0; xb < p.nxb; xb++)  // out-of-range rows / columns / channels are clipped by TMA
            ptx::tma_store_5d(&p.dense, A + (size_t)xb * p.R * 64 * 128, xb * 64, cb * 8, 0, y0, n);
        ptx::bulk_commit();
        ptx::bulk_wait_read0();   // shared memory must stay valid until the store has read it
    }
}

// ---------------------------------------------------------------------------------------------- host
static PFN_cuTensorMapEncodeTiled_v12000 get_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    if (!enc) {
        cudaDriverEntryPointQueryResult qr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &qr) != cudaSuccess) enc = nullptr;
    }
    return enc;
}

static int ilog2i(int v) {
    int r = 0;
    while ((1 << r) < v) r++;
    return (1 << r) == v ? r : -1;
}

// Returns true and launches when the layout is eligible; false = caller uses the generic kernels.
bool launch_convert_tma(const bdl_layout *l, const void *dense, void *bricked, cudaStream_t s, bool to_bricks,
                        bdl_status *st) {
    *st = BDL_OK;
    if (l->dtype != BDL_BF16 || l->nsp != 2 || l->C % 64 || l->Bn != 1 || l->brickmap) return false;
    if (ilog2i(l->Bh) < 0 || ilog2i(l->Bw) < 0 || l->Bw > 64 || 64 % l->Bw) return false;
    if (((uintptr_t)dense) % 16 || ((uintptr_t)bricked) % 16 || (l->W * 2) % 16) return false;
    const int W = (int)l->W, H = (int)l->H, C = (int)l->C, N = (int)l->N;
    const int nbx = (int)l->nb[3], nbh = (int)l->nb[2];
    const int Wg = nbx * l->Bw;
    if (Wg > 256 || nbx > 256 || Wg % 8) return false;
    PFN_cuTensorMapEncodeTiled_v12000 enc = get_encoder();
    if (!enc) return false;
    TmaConvParams P;
    memset(&P, 0, sizeof(P));
    P.N = N; P.C = C; P.H = H; P.W = W;
    P.Bh = l->Bh; P.Bw = l->Bw; P.lBh = ilog2i(l->Bh); P.lBw = ilog2i(l->Bw);
    P.nbx = nbx; P.nbh = nbh;
    P.nxb = (Wg + 63) / 64;
    P.ncb = C / 64;
    P.R = std::min(l->Bh, 2);   // small tiles: many CTAs per SM keep enough TMA traffic in flight
    if (const char *e = getenv("BDL_BRICKIFY_R")) P.R = std::max(1, std::min(l->Bh, atoi(e)));   // A/B knob
    while ((nbh * l->Bh) % P.R) P.R--;
    // dense NCHW viewed as (W, C/8, 8, H, N) with c = 8g + k: the box lands as [row][k][g][x]
    {
        const cuuint64_t plane = (cuuint64_t)H * W * 2;
        cuuint64_t dims[5] = {(cuuint64_t)W, (cuuint64_t)C / 8, 8, (cuuint64_t)H, (cuuint64_t)N};
        cuuint64_t strides[4] = {plane * 8, plane, (cuuint64_t)W * 2, plane * C};
        cuuint32_t box[5] = {64, 8, 8, (cuuint32_t)P.R, 1};
        cuuint32_t es[5] = {1, 1, 1, 1, 1};
        if (enc(&P.dense, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, const_cast<void *>(dense), dims, strides, box, es,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return false;
    }
    // bricks: (ch, xin, bx, yin, brick row over (n, by))
    {
        const cuuint64_t px = (cuuint64_t)l->c_pad * 2, brick = (cuuint64_t)l->brick_elems * 2;
        cuuint64_t dims[5] = {(cuuint64_t)l->c_pad, (cuuint64_t)l->Bw, (cuuint64_t)nbx, (cuuint64_t)l->Bh,
                              (cuuint64_t)(l->nb[0] * nbh)};
        cuuint64_t strides[4] = {px, brick, px * l->Bw, brick * nbx};
        cuuint32_t box[5] = {64, (cuuint32_t)l->Bw, (cuuint32_t)nbx, 1, 1};
        cuuint32_t es[5] = {1, 1, 1, 1, 1};
        if (enc(&P.bricks, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, bricked, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return false;
    }
    const size_t smem = (size_t)P.nxb * P.R * 64 * 128 + (size_t)P.R * Wg * 128;
    if (smem > 200 * 1024) return false;
    if (to_bricks) {
        P.out = bricked;
        P.Cp = (int)l->c_pad;
        P.brick_elems = l->brick_elems;
        const size_t smem_b = (size_t)P.nxb * P.R * 64 * 128;   // no staging tile: direct stores
        const long long grid = (long long)N * (nbh * l->Bh / P.R) * P.ncb;
        cudaFuncSetAttribute(brickify_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_b);
        cudaFuncSetAttribute(brickify_tma_kernel, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        brickify_tma_kernel<<<(unsigned)grid, 128, smem_b, s>>>(P);
    } else {
        const long long grid = (long long)N * ((H + P.R - 1) / P.R) * P.ncb;
        cudaFuncSetAttribute(unbrickify_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        launch_pdl(unbrickify_tma_kernel, dim3((unsigned)grid), dim3(128), smem, s, P);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) *st = fail(BDL_ECUDA, std::string("tma brickify: ") + cudaGetErrorString(e));
    return true;
}

}  // namespace bdl
