// Brick creation ("the cost of creating bricks, which is minimal") and its inverse.
// NC(D)HW dense  <->  bricked [phys][Bn][Bd][Bh][Bw][Cp] (include/brickdl.h).
//
// HBM-bound transposes.  One CTA owns a (sample n, brick-row bd/bh, channel group) tile spanning the
// full width W, staged in shared memory as [pixel][CGP] (channels innermost, CGP = CG + 1 elements):
//   dense side : every warp moves whole rows of one channel plane with 16-byte vectors (coalesced);
//   brick side : lanes walk the 16-byte channel vectors of consecutive pixels, so a warp writes or
//                reads 512 contiguous bytes of a brick per instruction.
// Index arithmetic is per 16-byte vector, never per element.
#include <algorithm>
#include <string>

#include "common.cuh"

namespace bdl {

struct ConvGeom {
    int CG, CGP, G;        // channels per tile, padded stride (elements), 16-B vectors per pixel
    int ngroups;
    int rows;              // Bd * Bh
    int Wfull;             // nb[3] * Bw
    int vec_ok;            // dense rows are 16-byte aligned (W * elem % 16 == 0)
};

template <typename T>
__global__ void __launch_bounds__(256) brickify_kernel(TView v, const T *__restrict__ src, ConvGeom cg) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T *tile = reinterpret_cast<T *>(smem_raw);
    constexpr int V = 16 / sizeof(T);
    const int g = blockIdx.x % cg.ngroups;
    int rest = blockIdx.x / cg.ngroups;
    const int bh = rest % v.nb[2];
    rest /= v.nb[2];
    const int bd = rest % v.nb[1];
    const int n = rest / v.nb[1];  // 0 .. nb[0]*Bn - 1
    const int Bd = v.B[1], Bh = v.B[2], W = v.ext[3], Wfull = cg.Wfull;
    const int c0 = g * cg.CG;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32, nwarps = blockDim.x / 32;
    const long long plane = (long long)v.ext[1] * v.ext[2] * W;
    // ---- phase 1: dense rows (channel c, depth z, row y) -> tile[pixel][c]; 4 vectors in flight/thread
    const int nrows = cg.CG * cg.rows;
    if (cg.vec_ok) {
        const int nvec = (Wfull + V - 1) / V;
        const int total = nrows * nvec;
        for (int i0 = threadIdx.x; i0 < total; i0 += 4 * blockDim.x) {
            uint4 u[4];
            int row_i[4], x_i[4];
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const int i = i0 + q * blockDim.x;
                row_i[q] = -1;
                u[q] = make_uint4(0, 0, 0, 0);
                if (i < total) {
                    const int r = i / nvec, x0 = (i - r * nvec) * V;
                    const int c = r / cg.rows, zy = r - c * cg.rows;
                    const int z = zy / Bh, y = zy - z * Bh;
                    const int d = bd * Bd + z, h = bh * Bh + y, cc = c0 + c;
                    row_i[q] = r;
                    x_i[q] = x0;
                    if (n < v.ext[0] && cc < v.C && d < v.ext[1] && h < v.ext[2] && x0 < W)
                        u[q] = __ldg(reinterpret_cast<const uint4 *>(src + ((long long)n * v.C + cc) * plane +
                                                                     ((long long)d * v.ext[2] + h) * W + x0));
                }
            }
#pragma unroll
            for (int q = 0; q < 4; q++) {
                if (row_i[q] < 0) continue;
                const int r = row_i[q], c = r / cg.rows, zy = r - c * cg.rows;
                T *trow = tile + (size_t)zy * Wfull * cg.CGP + c;
                const T *e = reinterpret_cast<const T *>(&u[q]);
#pragma unroll
                for (int k = 0; k < V; k++)
                    if (x_i[q] + k < Wfull) trow[(size_t)(x_i[q] + k) * cg.CGP] = e[k];
            }
        }
    } else {
        for (int r = warp; r < nrows; r += nwarps) {
            const int c = r / cg.rows, zy = r - c * cg.rows;
            const int z = zy / Bh, y = zy - z * Bh;
            const int d = bd * Bd + z, h = bh * Bh + y, cc = c0 + c;
            const bool rok = n < v.ext[0] && cc < v.C && d < v.ext[1] && h < v.ext[2];
            const T *row = src + ((long long)n * v.C + cc) * plane + ((long long)d * v.ext[2] + h) * W;
            T *trow = tile + (size_t)zy * Wfull * cg.CGP + c;
            for (int x = lane; x < Wfull; x += 32) trow[(size_t)x * cg.CGP] = (rok && x < W) ? row[x] : from_f<T>(0.f);
        }
    }
    __syncthreads();
    // ---- phase 2: brick pixels, 16-byte channel vectors, lanes fastest over the vectors of a pixel
    T *dst = reinterpret_cast<T *>(v.ptr);
    const int bn = n / v.B[0], nin = n - bn * v.B[0];
    const int npix = cg.rows * Wfull;
    const int gv = cg.CG / V;  // vectors of this group per pixel
    for (int i = threadIdx.x; i < npix * gv; i += blockDim.x) {
        const int q = i % gv, p = i / gv;
        const int zy = p / Wfull, x = p - zy * Wfull;
        const int z = zy / Bh, y = zy - z * Bh;
        const int bw = x / v.B[3], xi = x - bw * v.B[3];
        const long long logical = (((long long)bn * v.nb[1] + bd) * v.nb[2] + bh) * v.nb[3] + bw;
        const int inner = ((nin * Bd + z) * Bh + y) * v.B[3] + xi;
        const T *s = tile + (size_t)p * cg.CGP + q * V;
        union { uint4 u; T e[V]; } pk;
#pragma unroll
        for (int e = 0; e < V; e++) pk.e[e] = s[e];
        *reinterpret_cast<uint4 *>(dst + tv_phys(v, logical) * v.brick_elems + (long long)inner * v.Cp + c0 + q * V) = pk.u;
    }
}

template <typename T>
__global__ void __launch_bounds__(256) unbrickify_kernel(TView v, T *__restrict__ dstd, ConvGeom cg) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T *tile = reinterpret_cast<T *>(smem_raw);
    constexpr int V = 16 / sizeof(T);
    const int g = blockIdx.x % cg.ngroups;
    int rest = blockIdx.x / cg.ngroups;
    const int bh = rest % v.nb[2];
    rest /= v.nb[2];
    const int bd = rest % v.nb[1];
    const int n = rest / v.nb[1];
    if (n >= v.ext[0]) return;
    const int Bd = v.B[1], Bh = v.B[2], W = v.ext[3], Wfull = cg.Wfull;
    const int c0 = g * cg.CG;
    const T *src = reinterpret_cast<const T *>(v.ptr);
    const int bn = n / v.B[0], nin = n - bn * v.B[0];
    const int npix = cg.rows * Wfull;
    const int gv = cg.CG / V;
    const int total = npix * gv;
    for (int i0 = threadIdx.x; i0 < total; i0 += 4 * blockDim.x) {
        uint4 u[4];
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const int i = i0 + j * blockDim.x;
            if (i >= total) continue;
            const int q = i % gv, p = i / gv;
            const int zy = p / Wfull, x = p - zy * Wfull;
            const int z = zy / Bh, y = zy - z * Bh;
            const int bw = x / v.B[3], xi = x - bw * v.B[3];
            const long long logical = (((long long)bn * v.nb[1] + bd) * v.nb[2] + bh) * v.nb[3] + bw;
            const int inner = ((nin * Bd + z) * Bh + y) * v.B[3] + xi;
            u[j] = __ldg(reinterpret_cast<const uint4 *>(src + tv_phys(v, logical) * v.brick_elems + (long long)inner * v.Cp + c0 + q * V));
        }
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const int i = i0 + j * blockDim.x;
            if (i >= total) continue;
            const int q = i % gv, p = i / gv;
            const T *e = reinterpret_cast<const T *>(&u[j]);
            T *s = tile + (size_t)p * cg.CGP + q * V;
#pragma unroll
            for (int k = 0; k < V; k++) s[k] = e[k];
        }
    }
    __syncthreads();
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32, nwarps = blockDim.x / 32;
    const long long plane = (long long)v.ext[1] * v.ext[2] * W;
    const int nrows = cg.CG * cg.rows;
    for (int r = warp; r < nrows; r += nwarps) {
        const int c = r / cg.rows, zy = r - c * cg.rows;
        const int z = zy / Bh, y = zy - z * Bh;
        const int d = bd * Bd + z, h = bh * Bh + y, cc = c0 + c;
        if (cc >= v.C || d >= v.ext[1] || h >= v.ext[2]) continue;
        T *row = dstd + ((long long)n * v.C + cc) * plane + ((long long)d * v.ext[2] + h) * W;
        const T *trow = tile + (size_t)zy * Wfull * cg.CGP + c;
        if (cg.vec_ok) {
            for (int x0 = lane * V; x0 < W; x0 += 32 * V) {
                union { uint4 u; T e[V]; } pk;
#pragma unroll
                for (int i = 0; i < V; i++) pk.e[i] = trow[(size_t)(x0 + i) * cg.CGP];
                *reinterpret_cast<uint4 *>(row + x0) = pk.u;
            }
        } else {
            for (int x = lane; x < W; x += 32) row[x] = trow[(size_t)x * cg.CGP];
        }
    }
}

static bdl_status launch_convert(const bdl_layout *l, const void *src, void *dst, void *stream, bool to_bricks) {
    if (!layout_valid(l) || !src || !dst) return fail(BDL_EINVAL, "brickify/unbrickify: bad layout or NULL pointer");
    TView v = make_view(*l, to_bricks ? dst : const_cast<void *>(src));
    const int E = l->elem_bytes, V = 16 / E;
    ConvGeom cg;
    cg.rows = l->Bd * l->Bh;
    cg.Wfull = (int)(l->nb[3] * l->Bw);
    cg.vec_ok = ((l->W * E) % 16 == 0) && (((uintptr_t)(to_bricks ? src : dst)) % 16 == 0);
    const size_t budget = 96 * 1024;
    // channel group: the largest divisor of c_pad that is a multiple of V and fits the budget
    cg.CG = V;
    for (int k = 1; k <= l->c_pad / V; k++) {
        int c = l->c_pad / k;
        if (l->c_pad % k || c % V) continue;
        if ((size_t)cg.rows * cg.Wfull * (c + 1) * E <= budget) { cg.CG = c; break; }
    }
    cg.CGP = cg.CG + 1;
    cg.G = cg.CG / V;
    cg.ngroups = (l->c_pad + cg.CG - 1) / cg.CG;
    if (l->c_pad % cg.CG) return fail(BDL_EUNSUPPORTED, "brickify: channel grouping");
    size_t smem = (size_t)cg.rows * cg.Wfull * cg.CGP * E;
    if (smem > 200 * 1024) return fail(BDL_EUNSUPPORTED, "brickify: brick row tile too large for shared memory");
    long long nrows = to_bricks ? l->nb[0] * (long long)l->Bn : l->N;
    long long grid = nrows * l->nb[1] * l->nb[2] * cg.ngroups;
    if (grid <= 0 || grid > 0x7fffffff) return fail(BDL_EINVAL, "brickify: grid size out of range");
    cudaStream_t s = (cudaStream_t)stream;
    if (l->dtype == BDL_F32) {
        if (to_bricks) {
            cudaFuncSetAttribute(brickify_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            brickify_kernel<float><<<(unsigned)grid, 256, smem, s>>>(v, (const float *)src, cg);
        } else {
            cudaFuncSetAttribute(unbrickify_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            unbrickify_kernel<float><<<(unsigned)grid, 256, smem, s>>>(v, (float *)dst, cg);
        }
    } else {
        if (to_bricks) {
            cudaFuncSetAttribute(brickify_kernel<__nv_bfloat16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            brickify_kernel<__nv_bfloat16><<<(unsigned)grid, 256, smem, s>>>(v, (const __nv_bfloat16 *)src, cg);
        } else {
            cudaFuncSetAttribute(unbrickify_kernel<__nv_bfloat16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            unbrickify_kernel<__nv_bfloat16><<<(unsigned)grid, 256, smem, s>>>(v, (__nv_bfloat16 *)dst, cg);
        }
    }
    BDL_CUDA_CHECK_LAUNCH(to_bricks ? "bdl_brickify" : "bdl_unbrickify");
    return BDL_OK;
}

}  // namespace bdl

extern "C" bdl_status bdl_brickify(const bdl_layout *l, const void *src, void *dst, void *stream) {
    return bdl::launch_convert(l, src, dst, stream, true);
}

extern "C" bdl_status bdl_unbrickify(const bdl_layout *l, const void *src, void *dst, void *stream) {
    return bdl::launch_convert(l, src, dst, stream, false);
}
