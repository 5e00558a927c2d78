// Brick creation ("the cost of creating bricks, which is minimal") and its inverse.
// NC(D)HW dense  <->  bricked [phys][Bn][Bd][Bh][Bw][Cp] (include/brickdl.h).
//
// HBM-bound transposes without shared memory.  A thread owns a V x V block (V = 16 B / element: 8 bf16
// or 4 fp32): V channels x V consecutive pixels of one row.  It loads V 16-byte row vectors (one per
// channel) from the dense tensor, transposes the block in registers, and stores V 16-byte channel
// vectors (one per pixel) into the bricks -- and the reverse for unbrickify.  Lanes are ordered with
// the channel group fastest, so a warp's brick-side accesses are whole 128-byte pixel rows (C = 64
// bf16) and its dense-side accesses are 64-byte runs of each channel plane.
#include <algorithm>
#include <cstdlib>
#include <string>

#include "common.cuh"

namespace bdl {

template <typename T>
struct Vec {
    static constexpr int V = 16 / sizeof(T);
    union {
        uint4 u;
        T e[V];
    };
};

struct ConvGeom {
    int G;         // channel groups (Cp / V)
    int XG;        // pixel groups per brick-grid row (ceil((nb3*Bw) / V))
    int rows;      // rows of the brick grid: nb0*Bn (samples, padded) x nb1*Bd x nb2*Bh
    int vec_ok;    // dense rows are 16-byte aligned and W % V == 0
};

// Element offset of the channel-0 slot of pixel (n, d, h, w) in the bricked tensor.
__device__ __forceinline__ long long brick_px(const TView &v, int n, int d, int h, int w) {
    const int bn = n / v.B[0], bd = d / v.B[1], bh = h / v.B[2], bw = w / v.B[3];
    const long long logical = (((long long)bn * v.nb[1] + bd) * v.nb[2] + bh) * v.nb[3] + bw;
    const int inner = (((n - bn * v.B[0]) * v.B[1] + (d - bd * v.B[1])) * v.B[2] + (h - bh * v.B[2])) * v.B[3] + (w - bw * v.B[3]);
    return tv_phys(v, logical) * v.brick_elems + (long long)inner * v.Cp;
}

template <typename T>
__global__ void __launch_bounds__(256) brickify_kernel(TView v, const T *__restrict__ src, ConvGeom cg) {
    constexpr int V = Vec<T>::V;
    pdl_launch_dependents();  // the merged subgraph kernel may start its prologue
    const long long units = (long long)cg.rows * cg.XG * cg.G;
    const int Dg = v.nb[1] * v.B[1], Hg = v.nb[2] * v.B[2], Wg = v.nb[3] * v.B[3];
    const long long plane = (long long)v.ext[1] * v.ext[2] * v.ext[3];
    T *dst = reinterpret_cast<T *>(v.ptr);
    for (long long u = blockIdx.x * (long long)blockDim.x + threadIdx.x; u < units; u += (long long)gridDim.x * blockDim.x) {
        const int g = (int)(u % cg.G);
        long long r = u / cg.G;
        const int xg = (int)(r % cg.XG);
        r /= cg.XG;
        const int h = (int)(r % Hg);
        r /= Hg;
        const int d = (int)(r % Dg);
        const int n = (int)(r / Dg);
        const int x0 = xg * V, c0 = g * V;
        const bool row_ok = n < v.ext[0] && d < v.ext[1] && h < v.ext[2];
        Vec<T> in[V];
#pragma unroll
        for (int k = 0; k < V; k++) {
            const int c = c0 + k;
            const T *row = src + ((long long)n * v.C + c) * plane + ((long long)d * v.ext[2] + h) * v.ext[3];
            if (cg.vec_ok) {
                in[k].u = (row_ok && c < v.C && x0 < v.ext[3]) ? __ldg(reinterpret_cast<const uint4 *>(row + x0))
                                                              : make_uint4(0, 0, 0, 0);
            } else {
#pragma unroll
                for (int i = 0; i < V; i++)
                    in[k].e[i] = (row_ok && c < v.C && x0 + i < v.ext[3]) ? row[x0 + i] : from_f<T>(0.f);
            }
        }
#pragma unroll
        for (int i = 0; i < V; i++) {
            if (x0 + i >= Wg) break;
            Vec<T> o;
#pragma unroll
            for (int k = 0; k < V; k++) o.e[k] = in[k].e[i];
            *reinterpret_cast<uint4 *>(dst + brick_px(v, n, d, h, x0 + i) + c0) = o.u;
        }
    }
}

template <typename T>
__global__ void __launch_bounds__(256) unbrickify_kernel(TView v, T *__restrict__ dstd, ConvGeom cg) {
    constexpr int V = Vec<T>::V;
    pdl_wait();  // launched with PDL after the subgraph kernel: wait for its results
    const int XGd = (v.ext[3] + V - 1) / V;
    const long long units = (long long)v.ext[0] * v.ext[1] * v.ext[2] * XGd * cg.G;
    const long long plane = (long long)v.ext[1] * v.ext[2] * v.ext[3];
    const T *src = reinterpret_cast<const T *>(v.ptr);
    for (long long u = blockIdx.x * (long long)blockDim.x + threadIdx.x; u < units; u += (long long)gridDim.x * blockDim.x) {
        const int g = (int)(u % cg.G);
        long long r = u / cg.G;
        const int xg = (int)(r % XGd);
        r /= XGd;
        const int h = (int)(r % v.ext[2]);
        r /= v.ext[2];
        const int d = (int)(r % v.ext[1]);
        const int n = (int)(r / v.ext[1]);
        const int x0 = xg * V, c0 = g * V;
        Vec<T> in[V];
#pragma unroll
        for (int i = 0; i < V; i++)
            in[i].u = (x0 + i < v.ext[3]) ? __ldg(reinterpret_cast<const uint4 *>(src + brick_px(v, n, d, h, x0 + i) + c0))
                                          : make_uint4(0, 0, 0, 0);
#pragma unroll
        for (int k = 0; k < V; k++) {
            const int c = c0 + k;
            if (c >= v.C) break;
            T *row = dstd + ((long long)n * v.C + c) * plane + ((long long)d * v.ext[2] + h) * v.ext[3];
            Vec<T> o;
#pragma unroll
            for (int i = 0; i < V; i++) o.e[i] = in[i].e[k];
            if (cg.vec_ok) {
                *reinterpret_cast<uint4 *>(row + x0) = o.u;
            } else {
#pragma unroll
                for (int i = 0; i < V; i++)
                    if (x0 + i < v.ext[3]) row[x0 + i] = o.e[i];
            }
        }
    }
}

// Unbrickify of maps whose rows are not whole 16-B vectors (W % V != 0: ResNet-50's and VGG-16's 7 x 7 outputs):
// a CTA takes kSmallPx pixels of one sample's (D, H, W) volume x 128 bytes of channels, reads each pixel's channel
// run (coalesced: channels are innermost in a brick) into shared memory, and writes every channel's pixel run
// contiguously (consecutive threads -> consecutive pixels of one channel plane).  The register-transpose kernel
// wrote 2-byte scattered stores there (0.47 TB/s on ResNet-50's output).
constexpr int kSmallPx = 256;
template <typename T>
__global__ void __launch_bounds__(256) unbrickify_small_kernel(TView v, T *__restrict__ dstd) {
    constexpr int CB = 128 / sizeof(T);   // channels per block (128 B per pixel)
    __shared__ T tile[kSmallPx][CB + 2];  // (+2: consecutive pixels in different banks)
    pdl_wait();
    const long long vol = (long long)v.ext[1] * v.ext[2] * v.ext[3];
    const int nchunk = (int)((vol + kSmallPx - 1) / kSmallPx), ncb = (v.Cp + CB - 1) / CB;
    long long bid = blockIdx.x;
    const int cb = (int)(bid % ncb);
    bid /= ncb;
    const int chunk = (int)(bid % nchunk);
    const int n = (int)(bid / nchunk);
    const long long p0 = (long long)chunk * kSmallPx;
    const int np = (int)std::min<long long>(kSmallPx, vol - p0);
    const T *src = reinterpret_cast<const T *>(v.ptr);
    constexpr int V = 16 / sizeof(T);
    for (int i = threadIdx.x; i < np * (CB / V); i += blockDim.x) {   // 16-B chunks of each pixel's channel run
        const int px = i / (CB / V), q = i % (CB / V);
        const long long p = p0 + px;
        const int w = (int)(p % v.ext[3]), h = (int)((p / v.ext[3]) % v.ext[2]), d = (int)(p / ((long long)v.ext[3] * v.ext[2]));
        const int c = cb * CB + q * V;
        Vec<T> val;
        val.u = c < v.Cp ? __ldg(reinterpret_cast<const uint4 *>(src + brick_px(v, n, d, h, w) + c)) : make_uint4(0, 0, 0, 0);
#pragma unroll
        for (int e = 0; e < V; e++) tile[px][q * V + e] = val.e[e];
    }
    __syncthreads();
    const int nc = min(CB, v.C - cb * CB);
    for (int i = threadIdx.x; i < nc * np; i += blockDim.x) {
        const int c = i / np, px = i % np;
        dstd[((long long)n * v.C + cb * CB + c) * vol + p0 + px] = tile[px][c];
    }
}

bool launch_convert_tma(const bdl_layout *l, const void *dense, void *bricked, cudaStream_t s, bool to_bricks,
                        bdl_status *st);

static bdl_status launch_convert(const bdl_layout *l, const void *src, void *dst, void *stream, bool to_bricks) {
    if (!layout_valid(l) || !src || !dst) return fail(BDL_EINVAL, "brickify/unbrickify: bad layout or NULL pointer");
    {   // bf16, C % 64 == 0, identity BrickMap: TMA-staged transposes
        static const bool off = getenv("BDL_NO_TMA_BRICKIFY") != nullptr;
        bdl_status st;
        if (!off && launch_convert_tma(l, to_bricks ? src : dst, to_bricks ? dst : const_cast<void *>(src),
                                       (cudaStream_t)stream, to_bricks, &st))
            return st;
    }
    TView v = make_view(*l, to_bricks ? dst : const_cast<void *>(src));
    const int E = l->elem_bytes, V = 16 / E;
    ConvGeom cg;
    cg.G = l->c_pad / V;
    const long long Wg = l->nb[3] * l->Bw;
    cg.XG = (int)((Wg + V - 1) / V);
    cg.rows = (int)(l->nb[0] * l->Bn * l->nb[1] * l->Bd * l->nb[2] * l->Bh);
    cg.vec_ok = ((l->W % V) == 0) && (((uintptr_t)(to_bricks ? src : dst)) % 16 == 0);
    const long long units = to_bricks ? (long long)cg.rows * cg.XG * cg.G
                                      : l->N * l->D * l->H * ((l->W + V - 1) / V) * (long long)cg.G;
    const int threads = 256;
    const long long blocks = std::max<long long>(1, std::min<long long>((units + threads - 1) / threads, 148LL * 16));
    cudaStream_t s = (cudaStream_t)stream;
    if (!to_bricks && !cg.vec_ok && l->Bn == 1) {   // rows that are not whole 16-B vectors: shared-memory transpose
        const long long vol = l->D * l->H * l->W;
        const int CB = 128 / E;
        const long long nb = l->N * ((vol + kSmallPx - 1) / kSmallPx) * ((l->c_pad + CB - 1) / CB);
        if (l->dtype == BDL_F32)
            launch_pdl(unbrickify_small_kernel<float>, dim3((unsigned)nb), dim3(threads), 0, s, v, (float *)dst);
        else
            launch_pdl(unbrickify_small_kernel<__nv_bfloat16>, dim3((unsigned)nb), dim3(threads), 0, s, v, (__nv_bfloat16 *)dst);
        BDL_CUDA_CHECK_LAUNCH("bdl_unbrickify");
        return BDL_OK;
    }
    if (l->dtype == BDL_F32) {
        if (to_bricks) brickify_kernel<float><<<(unsigned)blocks, threads, 0, s>>>(v, (const float *)src, cg);
        else launch_pdl(unbrickify_kernel<float>, dim3((unsigned)blocks), dim3(threads), 0, s, v, (float *)dst, cg);
    } else {
        if (to_bricks) brickify_kernel<__nv_bfloat16><<<(unsigned)blocks, threads, 0, s>>>(v, (const __nv_bfloat16 *)src, cg);
        else launch_pdl(unbrickify_kernel<__nv_bfloat16>, dim3((unsigned)blocks), dim3(threads), 0, s, v, (__nv_bfloat16 *)dst, cg);
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
