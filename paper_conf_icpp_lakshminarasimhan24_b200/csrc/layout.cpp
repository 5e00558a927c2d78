// Brick layout host logic: bdl_layout_init, BrickInfo adjacency, error plumbing.
// Brick / BrickMap / BrickInfo are the paper's three data structures (§3.3.4,
// L664-736, Fig 6); the storage order is described in include/brickdl.h.
#include <cstring>
#include <string>

#include "internal.h"

namespace bdl {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }

bdl_status fail(bdl_status s, const std::string &msg) {
    g_err = msg;
    return s;
}

bool layout_valid(const bdl_layout *l) {
    return l && (l->nsp == 2 || l->nsp == 3) && l->N > 0 && l->C > 0 && l->D > 0 && l->H > 0 &&
           l->W > 0 && l->Bn > 0 && l->Bd > 0 && l->Bh > 0 && l->Bw > 0 && l->nbricks > 0;
}

TView make_view(const bdl_layout &l, void *ptr) {
    TView v;
    v.ptr = ptr;
    v.ext[0] = (int)l.N; v.ext[1] = (int)l.D; v.ext[2] = (int)l.H; v.ext[3] = (int)l.W;
    v.C = (int)l.C; v.Cp = l.c_pad;
    v.B[0] = l.Bn; v.B[1] = l.Bd; v.B[2] = l.Bh; v.B[3] = l.Bw;
    for (int i = 0; i < 4; i++) v.nb[i] = (int)l.nb[i];
    v.bmap = l.brickmap;
    v.brick_elems = l.brick_elems;
    return v;
}

}  // namespace bdl

using namespace bdl;

extern "C" {

const char *bdl_last_error(void) { return g_err.c_str(); }

const char *bdl_version(void) { return "brickdl-b200 0.1 (sm_100a)"; }

void bdl_plan_opts_default(bdl_plan_opts *o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->delta_threshold = 0.10;   // L644's 15 %, recalibrated for these B200 kernels (brickdl.h)
    o->tau = 4096;               // L656, "tau = 2^12"
    o->bcand[0] = 4; o->bcand[1] = 8; o->bcand[2] = 16; o->bcand[3] = 32;  // L654
    o->onchip_budget = 0;
    o->force_mode = BDL_MODE_AUTO;
    o->force_brick = 0;
    o->max_subgraph_layers = 0;
    o->num_sms = 0;
}

bdl_status bdl_layout_init(bdl_layout *out, int32_t nsp, int64_t N, int64_t C, int64_t D, int64_t H,
                           int64_t W, int32_t Bn, int32_t Bd, int32_t Bh, int32_t Bw, int32_t dtype) {
    if (!out) return fail(BDL_EINVAL, "bdl_layout_init: out is NULL");
    if (nsp != 2 && nsp != 3) return fail(BDL_EINVAL, "bdl_layout_init: nsp must be 2 or 3");
    if (N <= 0 || C <= 0 || D <= 0 || H <= 0 || W <= 0)
        return fail(BDL_EINVAL, "bdl_layout_init: non-positive tensor extent");
    if (Bn <= 0 || Bd <= 0 || Bh <= 0 || Bw <= 0)
        return fail(BDL_EINVAL, "bdl_layout_init: non-positive brick extent");
    if (nsp == 2 && (D != 1 || Bd != 1)) return fail(BDL_EINVAL, "bdl_layout_init: 2-D needs D = 1, Bd = 1");
    if (dtype != BDL_F32 && dtype != BDL_BF16) return fail(BDL_EINVAL, "bdl_layout_init: unknown dtype");
    std::memset(out, 0, sizeof(*out));
    out->nsp = nsp;
    out->dtype = dtype;
    out->N = N; out->C = C; out->D = D; out->H = H; out->W = W;
    out->Bn = Bn; out->Bd = Bd; out->Bh = Bh; out->Bw = Bw;
    out->elem_bytes = dtype == BDL_F32 ? 4 : 2;
    int q = 16 / out->elem_bytes;  // channels per 16-byte vector
    out->c_pad = (int32_t)((C + q - 1) / q * q);
    out->nb[0] = (N + Bn - 1) / Bn;
    out->nb[1] = (D + Bd - 1) / Bd;
    out->nb[2] = (H + Bh - 1) / Bh;
    out->nb[3] = (W + Bw - 1) / Bw;
    out->nbricks = out->nb[0] * out->nb[1] * out->nb[2] * out->nb[3];
    out->brick_elems = (int64_t)Bn * Bd * Bh * Bw * out->c_pad;
    out->brick_bytes = out->brick_elems * out->elem_bytes;
    out->total_bytes = out->nbricks * out->brick_bytes;
    out->brickmap = nullptr;
    return BDL_OK;
}

bdl_status bdl_brickinfo(const bdl_layout *l, const int32_t *brickmap_host, int32_t *adj_out) {
    if (!layout_valid(l) || !adj_out) return fail(BDL_EINVAL, "bdl_brickinfo: bad layout or adj_out NULL");
    const int64_t nbd = l->nb[1], nbh = l->nb[2], nbw = l->nb[3];
    const int ndir = (l->nsp == 3 ? 27 : 9) - 1;
    const int dlo = l->nsp == 3 ? -1 : 0, dhi = l->nsp == 3 ? 1 : 0;
    const int64_t nb = nbd * nbh * nbw;
    if (brickmap_host) {  // must be a permutation
        std::vector<char> seen(nb, 0);
        for (int64_t i = 0; i < nb; i++) {
            int32_t p = brickmap_host[i];
            if (p < 0 || p >= nb || seen[p]) return fail(BDL_EINVAL, "bdl_brickinfo: brickmap is not a permutation");
            seen[p] = 1;
        }
    }
    for (int64_t bd = 0; bd < nbd; bd++)
        for (int64_t bh = 0; bh < nbh; bh++)
            for (int64_t bw = 0; bw < nbw; bw++) {
                int64_t lg = (bd * nbh + bh) * nbw + bw;
                int64_t phys = brickmap_host ? brickmap_host[lg] : lg;
                int k = 0;
                for (int ed = dlo; ed <= dhi; ed++)
                    for (int eh = -1; eh <= 1; eh++)
                        for (int ew = -1; ew <= 1; ew++) {
                            if (!ed && !eh && !ew) continue;
                            int64_t qd = bd + ed, qh = bh + eh, qw = bw + ew;
                            int32_t v = -1;
                            if (qd >= 0 && qd < nbd && qh >= 0 && qh < nbh && qw >= 0 && qw < nbw) {
                                int64_t ql = (qd * nbh + qh) * nbw + qw;
                                v = (int32_t)(brickmap_host ? brickmap_host[ql] : ql);
                            }
                            adj_out[phys * ndir + k++] = v;
                        }
            }
    return BDL_OK;
}

}  // extern "C"
