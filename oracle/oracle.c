/*
 * BrickDL CPU ORACLE -- TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  The product path (paper_conf_icpp_lakshminarasimhan24_b200/
 * and its CUDA library) never links, imports or calls it, and this file shares no code,
 * header, table or helper with csrc/.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, the ICPP'24 BrickDL paper):
 *   Merged execution only REORDERS the computation of a chain of layers over bricks
 *   (§3.2; "without per-op sync", L418-425) -- the result it must reach
 *   is therefore the plain layer-by-layer definition on the unbricked NC(D)HW tensor.
 *   This file writes that definition out, in fp64, with no blocking, fusion or reordering:
 *
 *   oracle_conv     : sliding-window weighted sum, "a kernel or filter slides over the input
 *                     data to perform localized element-wise multiplications" (L182-185),
 *                     zero padding at feature-map boundaries (L434-437).  Cross-correlation
 *                     (SURVEY Q9), stride s, padding p, dilation d:
 *                       y[n,co,o] = sum_{ci,t} w[co,ci,t] * x[n,ci, s*o - p + d*t]   (x = 0 outside)
 *                     output extent floor((I + 2p - d(k-1) - 1)/s) + 1.
 *   oracle_conv_transpose : transposed convolution (of the mergeable set, L378-385), the adjoint of the
 *                     convolution's map from x to y: every input element is scattered through the kernel,
 *                       y[n,co,s*i - p + d*t] += w[co,ci,t] * x[n,ci,i]   (positions outside the output ignored)
 *                     output extent (I-1)s - 2p + d(k-1) + 1.
 *   oracle_maxpool  : max over the window, out-of-range positions ignored,
 *                     padding factor = pool stride (L456-458).
 *   oracle_epilogue : bias -> residual add -> ReLU -> storage rounding.
 *   oracle_round_bf16 : round-to-nearest-even to bfloat16 (8-bit significand), used where a
 *                     configuration stores activations in bf16 (north_star).
 *   oracle_brickify / oracle_unbrickify : the brick layout definition (L664-671):
 *                     fixed-size blocks along batch and spatial dims (never channels, L374-376),
 *                     row-major inside the brick, channels innermost, partial bricks and padded
 *                     channels zero ("masked ... with zero-valued elements", L742-743).
 *   oracle_brickinfo : BrickInfo adjacency (L680-684, Fig 6c): physical index of each
 *                     logical neighbour in direction order, via the BrickMap (Fig 6b).
 *
 * Parity pins: tests/test_oracle.py (delta input, identity kernel, ones/ones border counts,
 * composed-kernel halo growth, Toeplitz brute force, torch fp64 library routine, shift
 * equivariance, Fig 6 golden).  No function in this file is "parity unpinned".
 */
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#include <string.h>

#define IDX5(a, b, c, d, e, B, C, D, E) ((((((size_t)(a) * (B) + (b)) * (C) + (c)) * (D) + (d)) * (E) + (e)))

/* Round a double to the nearest bfloat16 value (ties to even), returned as a double.
 * bfloat16 = 1 sign bit, 8 exponent bits, 7 stored significand bits (8 with the hidden bit). */
double oracle_round_bf16(double x) {
    if (x == 0.0 || isnan(x) || isinf(x)) return x;
    int e;
    double m = frexp(x, &e);          /* x = m * 2^e, 0.5 <= |m| < 1 */
    double scaled = ldexp(m, 8);      /* 128 <= |scaled| < 256: 8 significant bits left of the point */
    double r = nearbyint(scaled);     /* default rounding mode = round half to even */
    return ldexp(r, e - 8);
}

/* N-d convolution (cross-correlation). 2D callers pass D=1, kd=1, sd=1, pd=0, dd=1.
 * x: [N][Ci][D][H][W], w: [Co][Ci][kd][kh][kw], bias: [Co] or NULL, y: [N][Co][Do][Ho][Wo]. */
void oracle_conv(const double *x, int N, int Ci, int D, int H, int W,
                 const double *w, const double *bias, int Co,
                 int kd, int kh, int kw, int sd, int sh, int sw,
                 int pd, int ph, int pw, int dd, int dh, int dw,
                 double *y, int Do, int Ho, int Wo) {
#pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; n++) {
        for (int co = 0; co < Co; co++) {
            for (int od = 0; od < Do; od++)
            for (int oh = 0; oh < Ho; oh++)
            for (int ow = 0; ow < Wo; ow++) {
                double acc = bias ? bias[co] : 0.0;
                for (int ci = 0; ci < Ci; ci++)
                for (int td = 0; td < kd; td++) {
                    int id = sd * od - pd + dd * td;
                    if (id < 0 || id >= D) continue;
                    for (int th = 0; th < kh; th++) {
                        int ih = sh * oh - ph + dh * th;
                        if (ih < 0 || ih >= H) continue;
                        for (int tw = 0; tw < kw; tw++) {
                            int iw = sw * ow - pw + dw * tw;
                            if (iw < 0 || iw >= W) continue;
                            acc += w[IDX5(co, ci, td, th, tw, Ci, kd, kh, kw)] *
                                   x[IDX5(n, ci, id, ih, iw, Ci, D, H, W)];
                        }
                    }
                }
                y[IDX5(n, co, od, oh, ow, Co, Do, Ho, Wo)] = acc;
            }
        }
    }
}

/* N-d transposed convolution (scatter form).  x: [N][Ci][D][H][W], w: [Co][Ci][kd][kh][kw] (w[co][ci][t] carries
 * input channel ci to output channel co through tap t), bias: [Co] or NULL, y: [N][Co][Do][Ho][Wo]. */
void oracle_conv_transpose(const double *x, int N, int Ci, int D, int H, int W,
                           const double *w, const double *bias, int Co,
                           int kd, int kh, int kw, int sd, int sh, int sw,
                           int pd, int ph, int pw, int dd, int dh, int dw,
                           double *y, int Do, int Ho, int Wo) {
#pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; n++) {
        for (int co = 0; co < Co; co++) {
            for (size_t q = 0; q < (size_t)Do * Ho * Wo; q++)
                y[IDX5(n, co, 0, 0, 0, Co, Do, Ho, Wo) + q] = bias ? bias[co] : 0.0;
            for (int ci = 0; ci < Ci; ci++)
            for (int id = 0; id < D; id++)
            for (int ih = 0; ih < H; ih++)
            for (int iw = 0; iw < W; iw++) {
                double xv = x[IDX5(n, ci, id, ih, iw, Ci, D, H, W)];
                for (int td = 0; td < kd; td++) {
                    int od = sd * id - pd + dd * td;
                    if (od < 0 || od >= Do) continue;
                    for (int th = 0; th < kh; th++) {
                        int oh = sh * ih - ph + dh * th;
                        if (oh < 0 || oh >= Ho) continue;
                        for (int tw = 0; tw < kw; tw++) {
                            int ow = sw * iw - pw + dw * tw;
                            if (ow < 0 || ow >= Wo) continue;
                            y[IDX5(n, co, od, oh, ow, Co, Do, Ho, Wo)] +=
                                w[IDX5(co, ci, td, th, tw, Ci, kd, kh, kw)] * xv;
                        }
                    }
                }
            }
        }
    }
}

/* Max pooling; out-of-range window positions are ignored (-inf padding). */
void oracle_maxpool(const double *x, int N, int C, int D, int H, int W,
                    int kd, int kh, int kw, int sd, int sh, int sw, int pd, int ph, int pw,
                    double *y, int Do, int Ho, int Wo) {
#pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; n++)
        for (int c = 0; c < C; c++)
            for (int od = 0; od < Do; od++)
            for (int oh = 0; oh < Ho; oh++)
            for (int ow = 0; ow < Wo; ow++) {
                double m = -INFINITY;
                for (int td = 0; td < kd; td++) {
                    int id = sd * od - pd + td;
                    if (id < 0 || id >= D) continue;
                    for (int th = 0; th < kh; th++) {
                        int ih = sh * oh - ph + th;
                        if (ih < 0 || ih >= H) continue;
                        for (int tw = 0; tw < kw; tw++) {
                            int iw = sw * ow - pw + tw;
                            if (iw < 0 || iw >= W) continue;
                            double v = x[IDX5(n, c, id, ih, iw, C, D, H, W)];
                            if (v > m) m = v;
                        }
                    }
                }
                y[IDX5(n, c, od, oh, ow, C, Do, Ho, Wo)] = m;
            }
}

/* In-place epilogue on a layer output y (bias already added by oracle_conv):
 *   y += residual (if non-NULL);  y = max(y, 0) (if relu);  y = round(y) (round: 0 = fp64 kept,
 *   1 = bf16, 2 = fp32). */
void oracle_epilogue(double *y, const double *residual, size_t n, int relu, int round_mode) {
    for (size_t i = 0; i < n; i++) {
        double v = y[i];
        if (residual) v += residual[i];
        if (relu && v < 0.0) v = 0.0;
        if (round_mode == 1) v = oracle_round_bf16(v);
        else if (round_mode == 2) v = (double)(float)v;
        y[i] = v;
    }
}

/* Brick layout definition.
 * Logical tensor x[N][C][D][H][W]; bricks of extent (Bn, Bd, Bh, Bw) over (n, d, h, w);
 * nb = ceil-div counts; the logical brick index is row-major over (bn, bd, bh, bw);
 * brickmap[logical] = physical slot (NULL = identity).  Each physical brick stores
 * [Bn][Bd][Bh][Bw][Cp] with channels innermost; Cp >= C, padded channels zero; positions of a
 * partial brick outside the tensor are zero.  dst must hold nbricks * Bn*Bd*Bh*Bw*Cp doubles. */
void oracle_brickify(const double *x, int N, int C, int D, int H, int W,
                     int Bn, int Bd, int Bh, int Bw, int Cp, const int32_t *brickmap, double *dst) {
    int nbn = (N + Bn - 1) / Bn, nbd = (D + Bd - 1) / Bd, nbh = (H + Bh - 1) / Bh, nbw = (W + Bw - 1) / Bw;
    size_t nbricks = (size_t)nbn * nbd * nbh * nbw;
    size_t belems = (size_t)Bn * Bd * Bh * Bw * Cp;
    memset(dst, 0, nbricks * belems * sizeof(double));
    for (int n = 0; n < N; n++)
    for (int c = 0; c < C; c++)
    for (int d = 0; d < D; d++)
    for (int h = 0; h < H; h++)
    for (int w = 0; w < W; w++) {
        size_t logical = (((size_t)(n / Bn) * nbd + d / Bd) * nbh + h / Bh) * nbw + w / Bw;
        size_t phys = brickmap ? (size_t)brickmap[logical] : logical;
        size_t inner = ((((size_t)(n % Bn) * Bd + d % Bd) * Bh + h % Bh) * Bw + w % Bw) * Cp + c;
        dst[phys * belems + inner] = x[IDX5(n, c, d, h, w, C, D, H, W)];
    }
}

void oracle_unbrickify(const double *src, int N, int C, int D, int H, int W,
                       int Bn, int Bd, int Bh, int Bw, int Cp, const int32_t *brickmap, double *x) {
    int nbd = (D + Bd - 1) / Bd, nbh = (H + Bh - 1) / Bh, nbw = (W + Bw - 1) / Bw;
    size_t belems = (size_t)Bn * Bd * Bh * Bw * Cp;
    for (int n = 0; n < N; n++)
    for (int c = 0; c < C; c++)
    for (int d = 0; d < D; d++)
    for (int h = 0; h < H; h++)
    for (int w = 0; w < W; w++) {
        size_t logical = (((size_t)(n / Bn) * nbd + d / Bd) * nbh + h / Bh) * nbw + w / Bw;
        size_t phys = brickmap ? (size_t)brickmap[logical] : logical;
        size_t inner = ((((size_t)(n % Bn) * Bd + d % Bd) * Bh + h % Bh) * Bw + w % Bw) * Cp + c;
        x[IDX5(n, c, d, h, w, C, D, H, W)] = src[phys * belems + inner];
    }
}

/* BrickInfo adjacency (Fig 6c): for every logical brick, in PHYSICAL order, the physical index
 * of each of its 3^nsp - 1 logical neighbours, directions enumerated row-major over
 * (dd, di, dj) in {-1,0,1}^nsp skipping (0,...,0) -- exactly the order of Fig 6c
 * (di = -1,-1,-1,0,0,1,1,1; dj = -1,0,1,-1,1,-1,0,1).  -1 marks a neighbour outside the grid.
 * Grid of brick counts (nbd, nbh, nbw) of one sample (nbd = 1 for 2D).
 * adj: [nbricks][3^nsp - 1]. */
void oracle_brickinfo(int nsp, int nbd, int nbh, int nbw, const int32_t *brickmap, int32_t *adj) {
    int ndir = (nsp == 3 ? 27 : 9) - 1;
    int nb = nbd * nbh * nbw;
    for (int bd = 0; bd < nbd; bd++)
    for (int bh = 0; bh < nbh; bh++)
    for (int bw = 0; bw < nbw; bw++) {
        int logical = (bd * nbh + bh) * nbw + bw;
        int phys = brickmap ? brickmap[logical] : logical;
        int k = 0;
        for (int ed = (nsp == 3 ? -1 : 0); ed <= (nsp == 3 ? 1 : 0); ed++)
        for (int eh = -1; eh <= 1; eh++)
        for (int ew = -1; ew <= 1; ew++) {
            if (ed == 0 && eh == 0 && ew == 0) continue;
            int qd = bd + ed, qh = bh + eh, qw = bw + ew;
            int v = -1;
            if (qd >= 0 && qd < nbd && qh >= 0 && qh < nbh && qw >= 0 && qw < nbw) {
                int ql = (qd * nbh + qh) * nbw + qw;
                v = brickmap ? brickmap[ql] : ql;
            }
            adj[(size_t)phys * ndir + k++] = v;
        }
    }
    (void)nb;
}
