// Brick creation ("the cost of creating bricks, which is minimal") and its inverse.
// NC(D)HW dense  <->  bricked [phys][Bn][Bd][Bh][Bw][Cp] (include/brickdl.h).
// HBM-bound transposes: one CTA stages a (brick-row x full width x channel-group) tile in shared
// memory so that both the dense rows (along W) and the brick pixels (channels innermost) are
// accessed contiguously.
#include <string>

#include "common.cuh"

namespace bdl {

constexpr int kCG = 16;  // channels per tile

// tile = (n, bd, bh, channel group g) x all W.  smem [Bd][Bh][W][kCG+1]
template <typename T>
__global__ void __launch_bounds__(256) brickify_kernel(TView v, const T *__restrict__ src, int ngroups) {
    extern __shared__ unsigned char smem_raw[];
    T *tile = reinterpret_cast<T *>(smem_raw);
    const int CGP = kCG + 1;
    int g = blockIdx.x % ngroups;
    int rest = blockIdx.x / ngroups;
    int bh = rest % v.nb[2]; rest /= v.nb[2];
    int bd = rest % v.nb[1]; rest /= v.nb[1];
    int n = rest;  // 0 .. N_padded-1 (covers partial batch bricks)
    const int Bd = v.B[1], Bh = v.B[2], W = v.ext[3];
    const int Wfull = v.nb[3] * v.B[3];
    const int c0 = g * kCG;
    const long long plane = (long long)v.ext[1] * v.ext[2] * v.ext[3];
    // phase 1: coalesced reads along W
    int total = kCG * Bd * Bh * Wfull;
    for (int i = threadIdx.x; i < total; i += blockDim.x) {
        int x = i % Wfull;
        int t = i / Wfull;
        int y = t % Bh; t /= Bh;
        int z = t % Bd;
        int c = t / Bd;
        int d = bd * Bd + z, h = bh * Bh + y, cc = c0 + c;
        T val = from_f<T>(0.f);
        if (n < v.ext[0] && cc < v.C && d < v.ext[1] && h < v.ext[2] && x < W)
            val = src[((long long)n * v.C + cc) * plane + ((long long)d * v.ext[2] + h) * W + x];
        tile[((z * Bh + y) * Wfull + x) * CGP + c] = val;
    }
    __syncthreads();
    // phase 2: brick pixels, channels innermost
    int cg = min(kCG, v.Cp - c0);
    int total2 = v.nb[3] * Bd * Bh * v.B[3] * cg;
    T *dst = reinterpret_cast<T *>(v.ptr);
    int bn = n / v.B[0], nin = n - bn * v.B[0];
    for (int i = threadIdx.x; i < total2; i += blockDim.x) {
        int c = i % cg;
        int t = i / cg;
        int xi = t % v.B[3]; t /= v.B[3];
        int y = t % Bh; t /= Bh;
        int z = t % Bd;
        int bw = t / Bd;
        long long logical = (((long long)bn * v.nb[1] + bd) * v.nb[2] + bh) * v.nb[3] + bw;
        long long phys = tv_phys(v, logical);
        int inner = ((nin * Bd + z) * Bh + y) * v.B[3] + xi;
        dst[phys * v.brick_elems + (long long)inner * v.Cp + c0 + c] = tile[((z * Bh + y) * Wfull + bw * v.B[3] + xi) * CGP + c];
    }
}

template <typename T>
__global__ void __launch_bounds__(256) unbrickify_kernel(TView v, T *__restrict__ dstd, int ngroups) {
    extern __shared__ unsigned char smem_raw[];
    T *tile = reinterpret_cast<T *>(smem_raw);
    const int CGP = kCG + 1;
    int g = blockIdx.x % ngroups;
    int rest = blockIdx.x / ngroups;
    int bh = rest % v.nb[2]; rest /= v.nb[2];
    int bd = rest % v.nb[1]; rest /= v.nb[1];
    int n = rest;
    if (n >= v.ext[0]) return;
    const int Bd = v.B[1], Bh = v.B[2], W = v.ext[3];
    const int Wfull = v.nb[3] * v.B[3];
    const int c0 = g * kCG;
    int cg = min(kCG, v.C - c0);
    const T *src = reinterpret_cast<const T *>(v.ptr);
    int bn = n / v.B[0], nin = n - bn * v.B[0];
    int total2 = v.nb[3] * Bd * Bh * v.B[3] * cg;
    for (int i = threadIdx.x; i < total2; i += blockDim.x) {
        int c = i % cg;
        int t = i / cg;
        int xi = t % v.B[3]; t /= v.B[3];
        int y = t % Bh; t /= Bh;
        int z = t % Bd;
        int bw = t / Bd;
        long long logical = (((long long)bn * v.nb[1] + bd) * v.nb[2] + bh) * v.nb[3] + bw;
        long long phys = tv_phys(v, logical);
        int inner = ((nin * Bd + z) * Bh + y) * v.B[3] + xi;
        tile[((z * Bh + y) * Wfull + bw * v.B[3] + xi) * CGP + c] = src[phys * v.brick_elems + (long long)inner * v.Cp + c0 + c];
    }
    __syncthreads();
    const long long plane = (long long)v.ext[1] * v.ext[2] * v.ext[3];
    int total = cg * Bd * Bh * W;
    for (int i = threadIdx.x; i < total; i += blockDim.x) {
        int x = i % W;
        int t = i / W;
        int y = t % Bh; t /= Bh;
        int z = t % Bd;
        int c = t / Bd;
        int d = bd * Bd + z, h = bh * Bh + y;
        if (d < v.ext[1] && h < v.ext[2])
            dstd[((long long)n * v.C + c0 + c) * plane + ((long long)d * v.ext[2] + h) * W + x] = tile[((z * Bh + y) * Wfull + x) * CGP + c];
    }
}

static bdl_status launch_convert(const bdl_layout *l, const void *src, void *dst, void *stream, bool to_bricks) {
    if (!layout_valid(l) || !src || !dst) return fail(BDL_EINVAL, "brickify/unbrickify: bad layout or NULL pointer");
    TView v = make_view(*l, to_bricks ? dst : const_cast<void *>(src));
    int ngroups = (int)((to_bricks ? l->c_pad : l->C) + kCG - 1) / kCG;
    long long nrows = to_bricks ? l->nb[0] * (long long)l->Bn : l->N;
    long long grid = nrows * l->nb[1] * l->nb[2] * ngroups;
    size_t smem = (size_t)l->Bd * l->Bh * l->nb[3] * l->Bw * (kCG + 1) * l->elem_bytes;
    if (smem > 200 * 1024) return fail(BDL_EUNSUPPORTED, "brickify: brick row tile too large for shared memory");
    if (grid <= 0 || grid > 0x7fffffff) return fail(BDL_EINVAL, "brickify: grid size out of range");
    cudaStream_t s = (cudaStream_t)stream;
    if (l->dtype == BDL_F32) {
        if (to_bricks) {
            cudaFuncSetAttribute(brickify_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            brickify_kernel<float><<<(unsigned)grid, 256, smem, s>>>(v, (const float *)src, ngroups);
        } else {
            cudaFuncSetAttribute(unbrickify_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            unbrickify_kernel<float><<<(unsigned)grid, 256, smem, s>>>(v, (float *)dst, ngroups);
        }
    } else {
        if (to_bricks) {
            cudaFuncSetAttribute(brickify_kernel<__nv_bfloat16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            brickify_kernel<__nv_bfloat16><<<(unsigned)grid, 256, smem, s>>>(v, (const __nv_bfloat16 *)src, ngroups);
        } else {
            cudaFuncSetAttribute(unbrickify_kernel<__nv_bfloat16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            unbrickify_kernel<__nv_bfloat16><<<(unsigned)grid, 256, smem, s>>>(v, (__nv_bfloat16 *)dst, ngroups);
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
