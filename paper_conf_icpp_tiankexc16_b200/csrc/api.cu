// api.cu -- the C ABI declared in include/safara.h.
//
// Host-side responsibilities only: argument / descriptor validation (the
// `dim` and `small` clause checks that replace the paper's two-version kernel,
// PAPER.md L1275-1291), NPB set_constants for the coefficients, the TMA
// tensor map for u, the work decomposition, and the launch.  Every step of the
// pass itself runs in the kernel (rhs_kernel.cuh).  No exceptions escape, no
// host synchronisation happens in the compute calls, nothing is allocated.
#include <cudaTypedefs.h>

#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <cstdio>
#include <mutex>

#include "safara_internal.h"

#ifndef SAFARA_TMA_SPLIT
#define SAFARA_TMA_SPLIT 0
#endif

using namespace safara;

namespace {

constexpr int kMaxDevices = 64;

constexpr int kMaxChunks = 64;

struct DeviceState {
    bool ready = false;
    int sms = 0;
    int ctas_fast = 0, ctas_strict = 0;
    cudaFuncAttributes attr_fast[4]{}, attr_strict[4]{};
    cudaFuncAttributes attr_ws_fast[2]{}, attr_ws_strict[2]{};
    // copy engines for safara_rhs_host's H2D / D2H pipeline (created at init)
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    cudaEvent_t ev_h[kMaxChunks] = {}, ev_c[kMaxChunks] = {};
    // SAFARA_FLAG_PIPELINE: the previous pipelined host call (buffers, chunks,
    // layout, stream); its ev_c events mark when its kernels stopped reading
    struct {
        bool valid = false;
        const double *u = nullptr, *f = nullptr, *r = nullptr;
        int C = 0, nz = 0, sk = 0;
        void *stream = nullptr;
    } pipe;
};

DeviceState g_dev[kMaxDevices];

// Tuning knobs, read once at init from the environment (defaults are the
// measured best).  SAFARA_L2PROMO: TMA L2 promotion
// 0=none 1=64B 2=128B 3=256B.  SAFARA_CHUNK: planes per chunk of the
// chunk-major work order (0 = whole column).  SAFARA_SCHED: 0 = balanced
// contiguous ranges, 1 = lockstep (column tile, k-part) per CTA.
struct Tune {
    int l2promo = 3;  // 256 B (A/B: +0.3-0.4 % over none, profiles/ab_knobs_r01.txt)
    int chunk = 0;
    int sched = 1;  // 0 = balanced contiguous ranges, 1 = lockstep (column, k-part)
    int interleave = 1;  // lockstep CTA order: 1 = tile-major across CTAs, 0 = part-major
    int face_ctas = 1;   // boundary faces on the idle SMs' extra CTAs (else by compute CTAs)
    int min_planes = MIN_PLANES_PER_CTA;  // shortest k-run a CTA is given
    int peer_bias = 1;   // f2: planes the slab-end k-part gives up (its tail waits for a peer)
    int split_bias = 0;  // experiments: shift the lockstep k-split points (no peer)
    int peer_bias_maxpart = 6;  // peer_bias only for k-parts of at most this many planes
    int peer_timeout_ms = 30000;  // f2 flag waits: give up and trap after this long
    int ws = 1;  // warp-specialised kernel (rhs_ws.cuh) where it applies (0: round-1 kernel)
    int iface = 1;  // WS launches: edge column tiles write the i-face columns (SAFARA_IFACE)
} g_tune;

int env_int(const char *name, int dflt) {
    const char *v = std::getenv(name);
    return v && *v ? std::atoi(v) : dflt;
}
std::mutex g_mutex;
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;
std::atomic<int64_t> g_launches{0};

int current_device(int *dev) {
    if (cudaGetDevice(dev) != cudaSuccess) return SAFARA_ERR_CUDA;
    if (*dev < 0 || *dev >= kMaxDevices) return SAFARA_ERR_NO_DEVICE;
    if (!g_dev[*dev].ready) return SAFARA_ERR_NOT_INIT;
    return SAFARA_OK;
}

// Largest element offset reachable through the descriptor, in 64-bit.
long long max_offset(const safara_dims_t &d, int nzb) {
    return (long long)(d.nx - 1) + (long long)d.sy * (d.ny - 1) + (long long)d.sm * 4 +
           (long long)d.sk * (nzb - 1);
}

int validate(const safara_dims_t *d, int nzb) {
    if (!d) return SAFARA_ERR_ARG;
    if (d->nx < 6 || d->ny < 6 || d->nz < 6 || nzb < 1) return SAFARA_ERR_SHAPE;
    if (d->sy < d->nx || d->sm <= 0 || d->sk <= 0) return SAFARA_ERR_LAYOUT;
    // j must be the second-fastest dimension (the smem tile is [m][j][i]).
    if (d->sy >= d->sm || d->sy >= d->sk) return SAFARA_ERR_LAYOUT;
    // non-overlap: order (j, m, k) by stride; each stride >= previous span.
    long long s1 = d->sm, e1 = 5, s2 = d->sk, e2 = nzb;
    if (s1 > s2) { std::swap(s1, s2); std::swap(e1, e2); }
    if (s1 == s2) return SAFARA_ERR_LAYOUT;
    if (s1 < (long long)d->sy * d->ny) return SAFARA_ERR_LAYOUT;
    if (s2 < s1 * e1) return SAFARA_ERR_LAYOUT;
    // TMA: global strides must be multiples of 16 bytes.
    if ((d->sy & 1) || (d->sm & 1) || (d->sk & 1)) return SAFARA_ERR_ALIGN;
    if (max_offset(*d, nzb) >= (1LL << 31)) return SAFARA_ERR_TOO_LARGE;
    return SAFARA_OK;
}

bool overlaps(const void *a, long long abytes, const void *b, long long bbytes) {
    const uintptr_t a0 = (uintptr_t)a, b0 = (uintptr_t)b;
    return a0 < b0 + (uintptr_t)bbytes && b0 < a0 + (uintptr_t)abytes;
}

int check_ptrs(const double *u, long long ubytes, const double *f, long long fbytes,
               const double *r, long long rbytes) {
    if (!u || !f || !r) return SAFARA_ERR_ARG;
    if (((uintptr_t)u | (uintptr_t)f | (uintptr_t)r) & 15u) return SAFARA_ERR_ALIGN;
    if (overlaps(r, rbytes, u, ubytes) || overlaps(r, rbytes, f, fbytes)) return SAFARA_ERR_ARG;
    return SAFARA_OK;
}

void to_coef(const safara_coeffs_t &in, Coef &c) {
    c.dt = in.dt;
    c.dssp = in.dssp;
    c.c1 = in.c1;
    c.c2 = in.c2;
    c.c1c2 = in.c1 * in.c2;  // NAS set_constants: c1c2 = c1*c2
    c.t2[0] = in.tx2;
    c.t2[1] = in.ty2;
    c.t2[2] = in.tz2;
    for (int m = 0; m < 5; ++m) {
        c.d1[0][m] = in.dxt[m];
        c.d1[1][m] = in.dyt[m];
        c.d1[2][m] = in.dzt[m];
    }
    const double *con[3] = {in.xxcon, in.yycon, in.zzcon};
    for (int a = 0; a < 3; ++a) {
        c.con2[a] = con[a][1];
        c.con2x43[a] = con[a][1] * in.con43;  // NAS: xxcon2*con43*(...), left to right
        c.con3[a] = con[a][2];
        c.con4[a] = con[a][3];
        c.con5[a] = con[a][4];
    }
}

// 4-D tensor map over a field: dim0 = i, then (j, m, k) ordered by stride;
// box (box_x, box_y, 5, 1), so the smem tile is [m][j][i] for any stride order.
int encode_map(CUtensorMap *map, const double *base, const safara_dims_t &d, int nplanes,
               int box_x, int box_y, int *pos_j, int *pos_m, int *pos_k) {
    struct Ax { int which; long long stride, extent, box; } ax[3] = {
        {0, d.sy, d.ny, box_y}, {1, d.sm, 5, SAFARA_TMA_SPLIT ? 1 : 5}, {2, d.sk, nplanes, 1}};
    std::sort(ax, ax + 3, [](const Ax &a, const Ax &b) { return a.stride < b.stride; });
    cuuint64_t gdim[4] = {(cuuint64_t)d.nx, 0, 0, 0};
    cuuint64_t gstride[3];
    cuuint32_t box[4] = {(cuuint32_t)box_x, 0, 0, 0};
    cuuint32_t estride[4] = {1, 1, 1, 1};
    for (int t = 0; t < 3; ++t) {
        gdim[t + 1] = (cuuint64_t)ax[t].extent;
        gstride[t] = (cuuint64_t)ax[t].stride * sizeof(double);
        box[t + 1] = (cuuint32_t)ax[t].box;
        if (ax[t].which == 0) *pos_j = t + 1;
        if (ax[t].which == 1) *pos_m = t + 1;
        if (ax[t].which == 2) *pos_k = t + 1;
    }
    const CUtensorMapL2promotion promo[4] = {
        CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_64B,
        CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B};
    CUresult r = g_encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, const_cast<double *>(base), gdim,
                          gstride, box, estride, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_NONE, promo[g_tune.l2promo & 3],
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? SAFARA_OK : SAFARA_ERR_CUDA;
}

// f2 (safara_rhs_peer): where the planes beyond the slab come from.
struct PeerCfg {
    int pk_lo, pk_hi, lo_koff, hi_koff;
    const double *u_lo, *u_hi;
    unsigned long long *flags, *flags_lo, *flags_hi;
    unsigned long long epoch;
};

// Shared launch path.  u has nzu planes, u plane = k - k0 + ukoff; forcing
// and rhs start at global plane k0.  [ka0,kb0) U [ka1,kb1) are computed;
// boundary faces of local planes [fk_lo, fk_hi) are copied.
int launch(const double *u, const double *f, double *r, const safara_dims_t &d, int nzu, int nzf,
           int k0,
           int ukoff, int ka0, int kb0, int ka1, int kb1, int fk_lo, int fk_hi,
           const safara_coeffs_t *coeffs, int flags, cudaStream_t stream,
           double *aux = nullptr, int naux = 0, int ska = 0, const PeerCfg *peer = nullptr,
           double *norm_work = nullptr, double *norm_out = nullptr, bool *fused = nullptr) {
    int dev;
    int rc = current_device(&dev);
    if (rc) return rc;
    if (!coeffs) return SAFARA_ERR_ARG;
    if (flags & ~SAFARA_FLAG_STRICT) return SAFARA_ERR_ARG;
    const DeviceState &st = g_dev[dev];

    Params p;
    std::memset(&p, 0, sizeof(p));
    p.nx = d.nx; p.ny = d.ny; p.nz = d.nz;
    p.sy = d.sy; p.sm = d.sm; p.sk = d.sk;
    p.u_sy = p.f_sy = p.r_sy = d.sy;
    p.u_sm = p.f_sm = p.r_sm = d.sm;
    p.u_sk = p.f_sk = p.r_sk = d.sk;
    p.u_sy64 = p.f_sy64 = p.r_sy64 = d.sy;
    p.u_sm64 = p.f_sm64 = p.r_sm64 = d.sm;
    p.u_sk64 = p.f_sk64 = p.r_sk64 = d.sk;
    p.k0 = k0; p.ukoff = ukoff; p.nzu = nzu;
    p.ka0 = ka0; p.kb0 = std::max(ka0, kb0);
    p.ka1 = ka1; p.kb1 = std::max(ka1, kb1);
    p.n0 = p.kb0 - p.ka0;
    p.nplanes = p.n0 + (p.kb1 - p.ka1);
    p.ntx = (d.nx - 2 + TX - 1) / TX;
    p.nty = (d.ny - 2 + TY - 1) / TY;
    p.ncol = p.ntx * p.nty;
    const long long units = (long long)p.ncol * p.nplanes;
    if (units >= (1LL << 31)) return SAFARA_ERR_TOO_LARGE;
    p.units = (int)units;
    p.chunk = std::max(1, std::min(g_tune.chunk > 0 ? g_tune.chunk : p.nplanes, p.nplanes));
    p.fk_lo = fk_lo; p.fk_hi = fk_hi;
    p.u = u; p.f = f; p.r = r;
    p.aux = aux; p.naux = naux; p.ska = ska;
    p.pk_lo = -(1 << 30);
    p.pk_hi = 1 << 30;
    if (peer) {
        p.pk_lo = peer->pk_lo; p.pk_hi = peer->pk_hi;
        p.lo_koff = peer->lo_koff; p.hi_koff = peer->hi_koff;
        p.u_lo = peer->u_lo; p.u_hi = peer->u_hi;
        p.pflags = peer->flags; p.pflags_lo = peer->flags_lo; p.pflags_hi = peer->flags_hi;
        p.epoch = peer->epoch;
        p.peer_timeout_ns = (unsigned long long)g_tune.peer_timeout_ms * 1000000ull;
    }
    to_coef(*coeffs, p.c);

    const bool strict = (flags & SAFARA_FLAG_STRICT) != 0;
    const int per_sm = strict ? st.ctas_strict : st.ctas_fast;
    const long long max_ctas = (long long)std::max(per_sm, 1) * st.sms;
    long long ncta;
    long long parts = p.ncol > 0 ? max_ctas / p.ncol : 0;
    parts = std::min<long long>(parts, std::max(1, p.nplanes / g_tune.min_planes));
    // Lockstep only when it keeps >= 90% of the CTA slots busy (e.g. class C:
    // 70 column tiles x 2 parts = 140 of 148); otherwise balanced ranges.
    const bool lockstep = g_tune.sched == 1 && parts >= 1 && p.nplanes > 0 &&
                          (parts * p.ncol * 10 >= 9 * std::min<long long>(max_ctas, p.units));
    if (lockstep) {
        // Every CTA owns one (column tile, k-part) and all parts start
        // together, so neighbouring tiles read a plane's shared halo at the
        // same time and the second read hits L2.
        ncta = p.ncol * parts;
        p.parts = g_tune.interleave ? (int)parts : 0;
        // f2: the k-part ending at the slab end pulls the upper peer's planes
        // in its last two steps; give it fewer planes so it ends with the rest
        // (bench.py --slab-sim with the single-loop march: SP-B/8 0.71 -> 0.75,
        // SP-B/4 1.03 -> 1.05; on 10-plane parts (C/8) no bias is best,
        // profiles/slab_sim_r01.txt)
        if (peer && peer->u_hi != nullptr && p.parts > 1 &&
            p.nplanes / p.parts <= g_tune.peer_bias_maxpart)
            p.split_bias = std::min(g_tune.peer_bias, std::max(0, p.nplanes / p.parts - 2));
        else if (p.parts > 1)
            p.split_bias = std::max(-(int)(p.nplanes / p.parts) + 2,
                                    std::min(g_tune.split_bias, (int)(p.nplanes / p.parts) - 2));
    } else {
        ncta = (p.units + g_tune.min_planes - 1) / g_tune.min_planes;
        ncta = std::min(ncta, max_ctas);
    }
    if (ncta < 1) {
        if (fk_hi <= fk_lo) return SAFARA_OK;  // nothing to do
        ncta = std::min<long long>(max_ctas, 16);
    }
    p.ncta = (int)ncta;
    // SMs the compute grid leaves idle take the boundary faces -- unless the
    // aux fields are requested: then each face point also reads u and writes
    // naux strided values, too much for a handful of SMs, so every compute
    // CTA takes a share before its march
    const long long face_pts =
        (long long)(2 * d.nx + 2 * (d.ny - 2)) * (fk_hi - fk_lo) + 2LL * (d.nx - 2) * (d.ny - 2);
    if (g_tune.face_ctas < 0) {  // PROBE ONLY (SAFARA_FACE_CTAS=-1): boundary faces skipped
        p.fk_lo = p.fk_hi = 0;
        fk_lo = fk_hi = 0;
    }
    p.nface_cta = (g_tune.face_ctas > 0 && !aux && fk_hi > fk_lo && p.units > 0 && ncta < max_ctas)
                      ? (int)std::min<long long>({max_ctas - ncta, 32, (face_pts + 4095) / 4096})
                      : 0;

#ifdef SAFARA_STEPLOG
    {   // debug builds only: per-CTA step timestamps of the last launch
        static unsigned long long *sl = nullptr;
        static int nct2 = 0;
        static int kaa[1024];
        if (!sl) {
            cudaMalloc(&sl, 1024 * 128 * sizeof(unsigned long long));
            std::atexit([] {
                static unsigned long long h[1024 * 128];
                cudaDeviceSynchronize();
                cudaMemcpy(h, sl, sizeof(h), cudaMemcpyDeviceToHost);
                FILE *f = std::fopen("gpurun_out/steplog.txt", "w");
                if (f) {
                    for (int c = 0; c < nct2; ++c) {
                        std::fprintf(f, "%d", c);
                        for (int t = 0; t < 128; ++t) std::fprintf(f, " %llu", h[c * 128 + t]);
                        std::fprintf(f, "\n");
                    }
                    std::fclose(f);
                }
            });
        }
        cudaMemsetAsync(sl, 0, 1024 * 128 * sizeof(unsigned long long), stream);
        p.steplog = sl;
        nct2 = p.ncta + p.nface_cta;
        (void)kaa;
    }
#endif
#ifdef SAFARA_TIMELINE
    {   // debug builds only: a static per-CTA timestamp buffer, dumped at exit
        // the last 4 launches, ring-indexed by launch number; the dump lists
        // them oldest first as "launch cta start end smid|cycles<<16"
        static unsigned long long *buf = nullptr;
        static int nct = 0;
        static long long nl = 0;
        if (!buf) {
            cudaMalloc(&buf, 4 * 3 * 1024 * sizeof(unsigned long long));
            std::atexit([] {
                static unsigned long long h[4 * 3 * 1024];
                cudaDeviceSynchronize();
                cudaMemcpy(h, buf, sizeof(h), cudaMemcpyDeviceToHost);
                FILE *f = std::fopen("gpurun_out/timeline.txt", "w");
                if (f) {
                    for (long long l = std::max(0LL, nl - 4); l < nl; ++l) {
                        const unsigned long long *b = h + 3 * 1024 * (l % 4);
                        for (int c = 0; c < nct; ++c)
                            std::fprintf(f, "%lld %d %llu %llu %llu\n", l, c, b[3 * c], b[3 * c + 1],
                                         b[3 * c + 2]);
                    }
                    std::fclose(f);
                }
            });
        }
        p.dbg = buf + 3 * 1024 * (nl % 4);
        ++nl;
        nct = p.ncta + p.nface_cta;
    }
#endif
    CUtensorMap umap, fmap;
    int pj, pm, pk;
    rc = encode_map(&umap, u, d, nzu, UX, UY, &p.pos_j, &p.pos_m, &p.pos_k);
    if (rc) return rc;
    rc = encode_map(&fmap, f, d, nzf, FX, TY, &pj, &pm, &pk);
    if (rc) return rc;
    bool ud = true;
    for (int ax = 0; ax < 3; ++ax)
        for (int m = 1; m < 5; ++m) ud = ud && (p.c.d1[ax][m] == p.c.d1[ax][0]);
    // the warp-specialised kernel serves launches whose CTAs each own one
    // (column tile, k range) segment: lockstep over a single plane range,
    // without the f1 aux output or the f2 peer halo
    const bool ws = g_tune.ws && lockstep && p.parts > 0 && p.n0 == p.nplanes &&
                    !(peer && aux);
    p.iface_tiles = ws && !aux && g_tune.iface ? 1 : 0;

    // f1 fused rhs_norm: the warp-specialised kernel with NAS coefficients
    // writes per-CTA partial sums; otherwise the caller runs the two-pass norm
    if (fused) *fused = norm_work != nullptr && ws && ud;
    if (fused && *fused) {
        // work[0]: CTA counter (zero between passes), partials from work + 8
        p.norm_ctr = reinterpret_cast<unsigned long long *>(norm_work);
        p.norm_part = norm_work + 8;
        p.norm_out = norm_out;
        p.norm_npts = (double)(d.nx - 2) * (double)(d.ny - 2) * (double)(d.nz - 2);
    }
    cudaError_t e;
    if (ws)
        e = strict ? launch_rhs_ws_strict(umap, fmap, p, ud, stream)
                   : launch_rhs_ws_fast(umap, fmap, p, ud, stream);
    else
        e = strict ? launch_rhs_strict(umap, fmap, p, ud, stream)
                   : launch_rhs_fast(umap, fmap, p, ud, stream);
    if (e != cudaSuccess) return SAFARA_ERR_CUDA;
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return SAFARA_OK;
}

// f1 aux array: naux component blocks with the shared (sy, sm) strides; the
// plane stride is naux*sm when components sit inside a plane (canonical
// [k][m][j][i]) and sk when they are outermost (SP's [m][k][j][i]).
int aux_layout(const safara_dims_t &d, int naux, int nplanes, int *ska, long long *bytes) {
    if (naux != SAFARA_AUX_BT && naux != SAFARA_AUX_SP) return SAFARA_ERR_ARG;
    const long long sa = d.sm < d.sk ? (long long)naux * d.sm : (long long)d.sk;
    if (d.sm >= d.sk && d.sm < d.sk * (long long)nplanes) return SAFARA_ERR_LAYOUT;
    const long long maxo = (long long)(d.nx - 1) + (long long)d.sy * (d.ny - 1) +
                           (long long)d.sm * (naux - 1) + sa * (nplanes - 1);
    if (maxo >= (1LL << 31) || sa >= (1LL << 31)) return SAFARA_ERR_TOO_LARGE;
    *ska = (int)sa;
    *bytes = (maxo + 1) * (long long)sizeof(double);
    return SAFARA_OK;
}

int check_aux(const double *aux, long long abytes, const double *u, long long ubytes,
              const double *f, long long fbytes, const double *r, long long rbytes) {
    if (!aux) return SAFARA_ERR_ARG;
    if ((uintptr_t)aux & 7u) return SAFARA_ERR_ALIGN;
    if (overlaps(aux, abytes, u, ubytes) || overlaps(aux, abytes, f, fbytes) ||
        overlaps(aux, abytes, r, rbytes))
        return SAFARA_ERR_ARG;
    return SAFARA_OK;
}

}  // namespace

void safara::count_launches(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

extern "C" {

int safara_coeffs_nas(int nx, int ny, int nz, double dt, safara_coeffs_t *out) {
    if (!out) return SAFARA_ERR_ARG;
    if (nx < 2 || ny < 2 || nz < 2) return SAFARA_ERR_SHAPE;
    // NPB set_constants.f, library's own copy.
    const double c1 = 1.4, c2 = 0.4, c3 = 0.1, c4 = 1.0, c5 = 1.4;
    const double dnxm1 = 1.0 / (double)(nx - 1);
    const double dnym1 = 1.0 / (double)(ny - 1);
    const double dnzm1 = 1.0 / (double)(nz - 1);
    const double c1c5 = c1 * c5, c3c4 = c3 * c4;
    const double tx1 = 1.0 / (dnxm1 * dnxm1), tx2 = 1.0 / (2.0 * dnxm1), tx3 = 1.0 / dnxm1;
    const double ty1 = 1.0 / (dnym1 * dnym1), ty2 = 1.0 / (2.0 * dnym1), ty3 = 1.0 / dnym1;
    const double tz1 = 1.0 / (dnzm1 * dnzm1), tz2 = 1.0 / (2.0 * dnzm1), tz3 = 1.0 / dnzm1;
    const double dx = 0.75, dy = 0.75, dz = 1.0;  // dx1..dx5, dy1..dy5, dz1..dz5
    const double conz1 = 1.0 - c1c5, con43 = 4.0 / 3.0, con16 = 1.0 / 6.0;
    std::memset(out, 0, sizeof(*out));
    out->dt = dt;
    out->dssp = 0.25 * std::max(dx, std::max(dy, dz));
    out->c1 = c1;
    out->c2 = c2;
    out->con43 = con43;
    out->tx2 = tx2;
    out->ty2 = ty2;
    out->tz2 = tz2;
    for (int m = 0; m < 5; ++m) {
        out->dxt[m] = dx * tx1;
        out->dyt[m] = dy * ty1;
        out->dzt[m] = dz * tz1;
    }
    const double t3[3] = {tx3, ty3, tz3};
    double *con[3] = {out->xxcon, out->yycon, out->zzcon};
    for (int a = 0; a < 3; ++a) {
        const double c34 = c3c4 * t3[a];
        con[a][0] = c34 * con43 * t3[a];
        con[a][1] = c34 * t3[a];
        con[a][2] = c34 * conz1 * t3[a];
        con[a][3] = c34 * con16 * t3[a];
        con[a][4] = c34 * c1c5 * t3[a];
    }
    return SAFARA_OK;
}

int safara_rhs_init(int device) {
    std::lock_guard<std::mutex> lock(g_mutex);
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count < 1) return SAFARA_ERR_NO_DEVICE;
    if (device < 0 || device >= count || device >= kMaxDevices) return SAFARA_ERR_NO_DEVICE;
    if (g_dev[device].ready) return SAFARA_OK;
    g_tune.l2promo = env_int("SAFARA_L2PROMO", g_tune.l2promo);
    g_tune.chunk = env_int("SAFARA_CHUNK", g_tune.chunk);
    g_tune.sched = env_int("SAFARA_SCHED", g_tune.sched);
    g_tune.interleave = env_int("SAFARA_INTERLEAVE", g_tune.interleave);
    g_tune.face_ctas = env_int("SAFARA_FACE_CTAS", g_tune.face_ctas);
    g_tune.min_planes = std::max(1, env_int("SAFARA_MIN_PLANES", g_tune.min_planes));
    g_tune.peer_bias = std::max(0, env_int("SAFARA_PEER_BIAS", g_tune.peer_bias));
    g_tune.split_bias = env_int("SAFARA_SPLIT_BIAS", g_tune.split_bias);
    g_tune.peer_bias_maxpart = env_int("SAFARA_PEER_BIAS_MAXPART", g_tune.peer_bias_maxpart);
    g_tune.peer_timeout_ms = std::max(1, env_int("SAFARA_PEER_TIMEOUT_MS", g_tune.peer_timeout_ms));
    g_tune.ws = env_int("SAFARA_WS", g_tune.ws);
    g_tune.iface = env_int("SAFARA_IFACE", g_tune.iface);
    int major = 0, minor = 0, sms = 0;
    if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device) ||
        cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, device) ||
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device))
        return SAFARA_ERR_CUDA;
    if (major != 10 || minor != 0) return SAFARA_ERR_NO_DEVICE;  // sm_100a code only
    if (!g_encode) {
        void *fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) !=
                cudaSuccess ||
            q != cudaDriverEntryPointSuccess || !fn)
            return SAFARA_ERR_CUDA;
        g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    }
    int prev = 0;
    if (cudaGetDevice(&prev) != cudaSuccess) return SAFARA_ERR_CUDA;
    if (cudaSetDevice(device) != cudaSuccess) return SAFARA_ERR_CUDA;
    DeviceState st;
    st.sms = sms;
    cudaError_t e = setup_rhs_fast(&st.ctas_fast, st.attr_fast);
    if (e == cudaSuccess) e = setup_rhs_strict(&st.ctas_strict, st.attr_strict);
    if (e == cudaSuccess) e = setup_rhs_ws_fast(st.attr_ws_fast);
    if (e == cudaSuccess) e = setup_rhs_ws_strict(st.attr_ws_strict);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&st.h2d, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&st.d2h, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&st.ev_fork, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&st.ev_join, cudaEventDisableTiming);
    for (int c = 0; c < kMaxChunks && e == cudaSuccess; ++c) {
        e = cudaEventCreateWithFlags(&st.ev_h[c], cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&st.ev_c[c], cudaEventDisableTiming);
    }
    cudaSetDevice(prev);
    if (e != cudaSuccess) return SAFARA_ERR_CUDA;
    st.ready = true;
    g_dev[device] = st;
    return SAFARA_OK;
}

int safara_pitch(int nx) { return nx <= 0 ? 0 : ((nx + 7) / 8) * 8; }

int safara_dims_canonical(int nx, int ny, int nz, safara_dims_t *out) {
    if (!out) return SAFARA_ERR_ARG;
    if (nx < 1 || ny < 1 || nz < 1) return SAFARA_ERR_SHAPE;
    const long long sy = safara_pitch(nx), sm = sy * ny, sk = 5 * sm;
    if (sk * nz >= (1LL << 31)) return SAFARA_ERR_TOO_LARGE;
    out->nx = nx; out->ny = ny; out->nz = nz;
    out->sy = (int32_t)sy; out->sm = (int32_t)sm; out->sk = (int32_t)sk;
    return SAFARA_OK;
}

int safara_validate_dims(const safara_dims_t *dims, int nz_buf) { return validate(dims, nz_buf); }

int safara_rhs_ex(const double *u, const double *forcing, double *rhs, const safara_dims_t *dims,
                  const safara_coeffs_t *coeffs, int flags, void *stream) {
    int rc = validate(dims, dims ? dims->nz : 0);
    if (rc) return rc;
    const long long bytes = (max_offset(*dims, dims->nz) + 1) * (long long)sizeof(double);
    rc = check_ptrs(u, bytes, forcing, bytes, rhs, bytes);
    if (rc) return rc;
    const int nz = dims->nz;
    return launch(u, forcing, rhs, *dims, nz, nz, 0, 0, 1, nz - 1, 0, 0, 0, nz, coeffs, flags,
                  (cudaStream_t)stream);
}

int safara_rhs(const double *u, const double *forcing, double *rhs, int nx, int ny, int nz,
               const safara_coeffs_t *coeffs, void *stream) {
    safara_dims_t d;
    int rc = safara_dims_canonical(nx, ny, nz, &d);
    if (rc) return rc;
    return safara_rhs_ex(u, forcing, rhs, &d, coeffs, 0, stream);
}

static int slab_launch(const double *u_slab, const double *forcing_slab, double *rhs_slab,
                       const safara_dims_t *dims, int k0, int nzl, const safara_coeffs_t *coeffs,
                       int flags, int part, void *stream, double *aux, int naux, int ska,
                       const PeerCfg *peer = nullptr) {
    if (!dims) return SAFARA_ERR_ARG;
    if (part < SAFARA_PART_ALL || part > SAFARA_PART_EDGE) return SAFARA_ERR_ARG;
    if (nzl < 2 || k0 < 0 || k0 + nzl > dims->nz) return SAFARA_ERR_SHAPE;
    const int nzu = nzl + 4;
    int rc = validate(dims, nzu);
    if (rc) return rc;
    const long long ubytes = (max_offset(*dims, nzu) + 1) * (long long)sizeof(double);
    const long long fbytes = (max_offset(*dims, nzl) + 1) * (long long)sizeof(double);
    rc = check_ptrs(u_slab, ubytes, forcing_slab, fbytes, rhs_slab, fbytes);
    if (rc) return rc;
    const int lo = std::max(k0, 1), hi = std::min(k0 + nzl, dims->nz - 1);
    int ka0 = lo, kb0 = hi, ka1 = 0, kb1 = 0, fk_lo = 0, fk_hi = nzl;
    if (part == SAFARA_PART_INTERIOR) {
        ka0 = std::max(lo, k0 + 2);
        kb0 = std::min(hi, k0 + nzl - 2);
    } else if (part == SAFARA_PART_EDGE) {
        const int e0 = std::min(hi, k0 + 2);
        const int e1 = std::max(e0, std::max(lo, k0 + nzl - 2));
        ka0 = lo; kb0 = e0; ka1 = e1; kb1 = hi;
        fk_lo = fk_hi = 0;
    }
    return launch(u_slab, forcing_slab, rhs_slab, *dims, nzu, nzl, k0, 2, ka0, kb0, ka1, kb1, fk_lo,
                  fk_hi, coeffs, flags, (cudaStream_t)stream, aux, naux, ska, peer);
}

int safara_rhs_peer(const double *u_slab, const double *forcing_slab, double *rhs_slab,
                    const safara_dims_t *dims, int k0, int nzl, const safara_peer_t *peer,
                    const safara_coeffs_t *coeffs, int flags, void *stream) {
    if (!dims || !peer) return SAFARA_ERR_ARG;
    const bool has_lo = k0 > 0, has_hi = k0 + nzl < dims->nz;
    if ((peer->u_lo != nullptr) != has_lo || (peer->u_hi != nullptr) != has_hi)
        return SAFARA_ERR_ARG;
    // neighbours own >= 2 planes: [k0_lo, k0) and [k0_hi, ...)
    if (has_lo && !(peer->k0_lo <= k0 - 2 && peer->k0_lo >= 0)) return SAFARA_ERR_ARG;
    if (has_hi && peer->k0_hi != k0 + nzl) return SAFARA_ERR_ARG;
    if (((uintptr_t)peer->u_lo | (uintptr_t)peer->u_hi) & 15u) return SAFARA_ERR_ALIGN;
    if (peer->epoch) {
        if (!peer->flags || (peer->flags_lo != nullptr) != has_lo ||
            (peer->flags_hi != nullptr) != has_hi)
            return SAFARA_ERR_ARG;
        if (((uintptr_t)peer->flags | (uintptr_t)peer->flags_lo | (uintptr_t)peer->flags_hi) & 7u)
            return SAFARA_ERR_ALIGN;
    }
    PeerCfg pc;
    pc.pk_lo = has_lo ? k0 : -(1 << 30);
    pc.pk_hi = has_hi ? k0 + nzl : 1 << 30;
    pc.lo_koff = has_lo ? 2 - peer->k0_lo : 0;  // neighbour local plane = k - k0_lo + 2
    pc.hi_koff = has_hi ? 2 - peer->k0_hi : 0;
    pc.u_lo = peer->u_lo;
    pc.u_hi = peer->u_hi;
    pc.flags = reinterpret_cast<unsigned long long *>(peer->flags);
    pc.flags_lo = reinterpret_cast<unsigned long long *>(peer->flags_lo);
    pc.flags_hi = reinterpret_cast<unsigned long long *>(peer->flags_hi);
    pc.epoch = peer->epoch;
    return slab_launch(u_slab, forcing_slab, rhs_slab, dims, k0, nzl, coeffs, flags,
                       SAFARA_PART_ALL, stream, nullptr, 0, 0, &pc);
}

int safara_ipc_get(const void *dptr, void *handle, int64_t *offset) {
    if (!dptr || !handle || !offset) return SAFARA_ERR_ARG;
    static PFN_cuMemGetAddressRange_v3020 range = nullptr;
    if (!range) {
        void *fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) !=
                cudaSuccess || !fn)
            return SAFARA_ERR_CUDA;
        range = (PFN_cuMemGetAddressRange_v3020)fn;
    }
    CUdeviceptr base = 0;
    size_t size = 0;
    if (range(&base, &size, (CUdeviceptr)dptr) != CUDA_SUCCESS) {
        (void)cudaGetLastError();
        return SAFARA_ERR_CUDA;
    }
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, (void *)base) != cudaSuccess) {
        (void)cudaGetLastError();  // not sticky: do not leave it for a later call to report
        return SAFARA_ERR_CUDA;
    }
    static_assert(sizeof(h) == SAFARA_IPC_HANDLE_BYTES, "IPC handle size");
    std::memcpy(handle, &h, sizeof(h));
    *offset = (int64_t)((CUdeviceptr)dptr - base);
    return SAFARA_OK;
}

int safara_ipc_open(const void *handle, int64_t offset, void **dptr) {
    if (!handle || !dptr || offset < 0) return SAFARA_ERR_ARG;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, sizeof(h));
    void *base = nullptr;
    if (cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        (void)cudaGetLastError();
        return SAFARA_ERR_CUDA;
    }
    *dptr = (char *)base + offset;
    return SAFARA_OK;
}

int safara_ipc_close(void *dptr, int64_t offset) {
    if (!dptr || offset < 0) return SAFARA_ERR_ARG;
    return cudaIpcCloseMemHandle((char *)dptr - offset) == cudaSuccess ? SAFARA_OK
                                                                        : SAFARA_ERR_CUDA;
}

int safara_rhs_slab(const double *u_slab, const double *forcing_slab, double *rhs_slab,
                    const safara_dims_t *dims, int k0, int nzl, const safara_coeffs_t *coeffs,
                    int flags, int part, void *stream) {
    return slab_launch(u_slab, forcing_slab, rhs_slab, dims, k0, nzl, coeffs, flags, part, stream,
                       nullptr, 0, 0);
}

int safara_rhs_aux(const double *u, const double *forcing, double *rhs, double *aux, int naux,
                   const safara_dims_t *dims, const safara_coeffs_t *coeffs, int flags,
                   void *stream) {
    int rc = validate(dims, dims ? dims->nz : 0);
    if (rc) return rc;
    const long long bytes = (max_offset(*dims, dims->nz) + 1) * (long long)sizeof(double);
    rc = check_ptrs(u, bytes, forcing, bytes, rhs, bytes);
    if (rc) return rc;
    int ska;
    long long abytes;
    rc = aux_layout(*dims, naux, dims->nz, &ska, &abytes);
    if (rc) return rc;
    rc = check_aux(aux, abytes, u, bytes, forcing, bytes, rhs, bytes);
    if (rc) return rc;
    const int nz = dims->nz;
    return launch(u, forcing, rhs, *dims, nz, nz, 0, 0, 1, nz - 1, 0, 0, 0, nz, coeffs, flags,
                  (cudaStream_t)stream, aux, naux, ska);
}

int safara_rhs_fused(const double *u, const double *forcing, double *rhs, double *aux, int naux,
                     double *work, double *rms, const safara_dims_t *dims,
                     const safara_coeffs_t *coeffs, int flags, void *stream) {
    int rc = validate(dims, dims ? dims->nz : 0);
    if (rc) return rc;
    const long long bytes = (max_offset(*dims, dims->nz) + 1) * (long long)sizeof(double);
    rc = check_ptrs(u, bytes, forcing, bytes, rhs, bytes);
    if (rc) return rc;
    int ska = 0;
    if (aux) {
        long long abytes;
        rc = aux_layout(*dims, naux, dims->nz, &ska, &abytes);
        if (rc) return rc;
        rc = check_aux(aux, abytes, u, bytes, forcing, bytes, rhs, bytes);
        if (rc) return rc;
    } else {
        naux = 0;
    }
    if (rms) {
        if (!work) return SAFARA_ERR_ARG;
        if (((uintptr_t)work | (uintptr_t)rms) & 7u) return SAFARA_ERR_ALIGN;
        const long long wbytes = ((long long)safara_norm_work_doubles() + 8) * 8;
        if (overlaps(work, wbytes, rhs, bytes) || overlaps(work, wbytes, u, bytes) ||
            overlaps(work, wbytes, forcing, bytes) || overlaps(rms, 40, rhs, bytes) ||
            overlaps(rms, 40, work, wbytes))
            return SAFARA_ERR_ARG;
    }
    const int nz = dims->nz;
    bool fused = false;
    rc = launch(u, forcing, rhs, *dims, nz, nz, 0, 0, 1, nz - 1, 0, 0, 0, nz, coeffs, flags,
                (cudaStream_t)stream, aux, naux, ska, nullptr, rms ? work : nullptr, rms,
                rms ? &fused : nullptr);
    if (rc || !rms || fused) return rc;
    // not the warp-specialised NAS path: the two-pass norm (work[0] untouched)
    return safara_rhs_rms(rhs, dims, work + 8, rms, stream);
}

int safara_rhs_slab_aux(const double *u_slab, const double *forcing_slab, double *rhs_slab,
                        double *aux_slab, int naux, const safara_dims_t *dims, int k0, int nzl,
                        const safara_coeffs_t *coeffs, int flags, int part, void *stream) {
    if (!dims) return SAFARA_ERR_ARG;
    if (nzl < 2 || k0 < 0 || k0 + nzl > dims->nz) return SAFARA_ERR_SHAPE;
    int ska;
    long long abytes;
    int rc = aux_layout(*dims, naux, nzl, &ska, &abytes);
    if (rc) return rc;
    const long long ubytes = (max_offset(*dims, nzl + 4) + 1) * (long long)sizeof(double);
    const long long fbytes = (max_offset(*dims, nzl) + 1) * (long long)sizeof(double);
    rc = check_aux(aux_slab, abytes, u_slab, ubytes, forcing_slab, fbytes, rhs_slab, fbytes);
    if (rc) return rc;
    return slab_launch(u_slab, forcing_slab, rhs_slab, dims, k0, nzl, coeffs, flags, part, stream,
                       aux_slab, naux, ska);
}

int safara_rhs_host(const double *u_host, const double *forcing_host, double *rhs_host,
                    double *u_dev, double *forcing_dev, double *rhs_dev, int nx, int ny, int nz,
                    const safara_coeffs_t *coeffs, int flags, int nchunks, void *stream) {
    safara_dims_t d;
    int rc = safara_dims_canonical(nx, ny, nz, &d);
    if (rc) return rc;
    return safara_rhs_host_ex(u_host, forcing_host, rhs_host, u_dev, forcing_dev, rhs_dev, &d,
                              coeffs, flags, nchunks, stream);
}

int safara_rhs_host_ex(const double *u_host, const double *forcing_host, double *rhs_host,
                       double *u_dev, double *forcing_dev, double *rhs_dev,
                       const safara_dims_t *dims, const safara_coeffs_t *coeffs, int flags,
                       int nchunks, void *stream) {
    if (!u_host || !forcing_host || !rhs_host || !dims) return SAFARA_ERR_ARG;
    if (flags & ~(SAFARA_FLAG_STRICT | SAFARA_FLAG_PIPELINE)) return SAFARA_ERR_ARG;
    const bool pipeline = (flags & SAFARA_FLAG_PIPELINE) != 0;
    flags &= SAFARA_FLAG_STRICT;
    const safara_dims_t d = *dims;
    const int nz = d.nz;
    int rc = validate(&d, nz);
    if (rc) return rc;
    if ((long long)d.sk < 5LL * d.sm) return SAFARA_ERR_LAYOUT;  // k outermost: chunks are byte ranges
    const long long bytes = (long long)d.sk * nz * (long long)sizeof(double);
    rc = check_ptrs(u_dev, bytes, forcing_dev, bytes, rhs_dev, bytes);
    if (rc) return rc;
    int dev;
    rc = current_device(&dev);
    if (rc) return rc;
    DeviceState &st = g_dev[dev];
    std::lock_guard<std::mutex> lock(g_mutex);  // the copy streams/events are per device
    cudaStream_t s = (cudaStream_t)stream;
    // k-chunks of >= 4 planes; chunk c computes planes [z_c, z_{c+1}) once the
    // H2D of chunk c+1 (which holds its +2 ghost planes) has landed, and its
    // rhs planes go back while later chunks are copied in and computed.
    int C = std::max(1, std::min(std::min(nchunks, kMaxChunks), nz / 4));
    auto z = [&](int c) { return (int)((long long)nz * c / C); };
    const size_t plane = (size_t)d.sk * sizeof(double);
    // pipelined continuation of the previous call: no fork on `stream` (whose
    // tail is the previous call's D2H); each H2D chunk instead waits for the
    // previous call's kernels that read its planes (chunks c-1 .. c+1)
    const bool cont = pipeline && st.pipe.valid && st.pipe.u == u_dev &&
                      st.pipe.f == forcing_dev && st.pipe.r == rhs_dev && st.pipe.C == C &&
                      st.pipe.nz == nz && st.pipe.sk == d.sk && st.pipe.stream == stream;
    st.pipe.valid = false;  // set again only when this call is fully enqueued
    bool ok = cudaEventRecord(st.ev_fork, s) == cudaSuccess &&
              cudaStreamWaitEvent(st.d2h, st.ev_fork, 0) == cudaSuccess &&
              (cont || cudaStreamWaitEvent(st.h2d, st.ev_fork, 0) == cudaSuccess);
    for (int c = 0; ok && c < C; ++c) {
        const size_t off = (size_t)z(c) * d.sk, len = (size_t)(z(c + 1) - z(c)) * plane;
        if (cont) ok = cudaStreamWaitEvent(st.h2d, st.ev_c[std::min(c + 1, C - 1)], 0) == cudaSuccess;
        ok = ok && cudaMemcpyAsync(u_dev + off, u_host + off, len, cudaMemcpyHostToDevice, st.h2d) ==
                 cudaSuccess &&
             cudaMemcpyAsync(forcing_dev + off, forcing_host + off, len, cudaMemcpyHostToDevice,
                             st.h2d) == cudaSuccess &&
             cudaEventRecord(st.ev_h[c], st.h2d) == cudaSuccess;
    }
    for (int c = 0; ok && c < C; ++c) {
        ok = cudaStreamWaitEvent(s, st.ev_h[std::min(c + 1, C - 1)], 0) == cudaSuccess;
        if (!ok) break;
        rc = launch(u_dev, forcing_dev, rhs_dev, d, nz, nz, 0, 0, std::max(z(c), 1),
                    std::min(z(c + 1), nz - 1), 0, 0, z(c), z(c + 1), coeffs, flags, s);
        if (rc) return rc;
        const size_t off = (size_t)z(c) * d.sk, len = (size_t)(z(c + 1) - z(c)) * plane;
        ok = cudaEventRecord(st.ev_c[c], s) == cudaSuccess &&
             cudaStreamWaitEvent(st.d2h, st.ev_c[c], 0) == cudaSuccess &&
             cudaMemcpyAsync(rhs_host + off, rhs_dev + off, len, cudaMemcpyDeviceToHost,
                             st.d2h) == cudaSuccess;
    }
    ok = ok && cudaEventRecord(st.ev_join, st.d2h) == cudaSuccess &&
         cudaStreamWaitEvent(s, st.ev_join, 0) == cudaSuccess;
    st.pipe.valid = ok && pipeline;
    st.pipe.u = u_dev; st.pipe.f = forcing_dev; st.pipe.r = rhs_dev;
    st.pipe.C = C; st.pipe.nz = nz; st.pipe.sk = d.sk; st.pipe.stream = stream;
    return ok ? SAFARA_OK : SAFARA_ERR_CUDA;
}

int safara_norm_work_doubles(void) { return 5 * norm_grid(); }

// Shared by safara_rhs_sumsq / safara_rhs_rms: npts > 0 finishes rhs_norm.
static int sumsq_launch(const double *rhs, const safara_dims_t *dims, int k0, int nzl,
                        double *work, double *out, void *stream, double npts) {
    int dev;
    int rc = current_device(&dev);
    if (rc) return rc;
    if (!dims) return SAFARA_ERR_ARG;
    if (nzl < 1 || k0 < 0 || k0 + nzl > dims->nz) return SAFARA_ERR_SHAPE;
    rc = validate(dims, nzl);
    if (rc) return rc;
    if (!rhs || !work || !out) return SAFARA_ERR_ARG;
    if (((uintptr_t)rhs | (uintptr_t)work | (uintptr_t)out) & 7u) return SAFARA_ERR_ALIGN;
    const long long rbytes = (max_offset(*dims, nzl) + 1) * (long long)sizeof(double);
    const long long wbytes = (long long)safara_norm_work_doubles() * sizeof(double);
    if (overlaps(work, wbytes, rhs, rbytes) || overlaps(out, 40, rhs, rbytes) ||
        overlaps(out, 40, work, wbytes))
        return SAFARA_ERR_ARG;
    const int lo = std::max(k0, 1), hi = std::min(k0 + nzl, dims->nz - 1);
    const int nk = std::max(0, hi - lo);
    cudaError_t e = launch_sumsq(rhs, dims->nx, dims->ny, dims->sy, dims->sm, dims->sk, lo - k0,
                                 nk, work, out, (cudaStream_t)stream, npts);
    if (e != cudaSuccess) return SAFARA_ERR_CUDA;
    g_launches.fetch_add(2, std::memory_order_relaxed);
    return SAFARA_OK;
}

int safara_rhs_sumsq(const double *rhs, const safara_dims_t *dims, int k0, int nzl, double *work,
                     double *out, void *stream) {
    return sumsq_launch(rhs, dims, k0, nzl, work, out, stream, 0.0);
}

int safara_rhs_rms(const double *rhs, const safara_dims_t *dims, double *work, double *rms,
                   void *stream) {
    if (!dims) return SAFARA_ERR_ARG;
    const double npts = (double)(dims->nx - 2) * (double)(dims->ny - 2) * (double)(dims->nz - 2);
    return sumsq_launch(rhs, dims, 0, dims->nz, work, rms, stream, npts);
}

int safara_seismic_dz(const double *vz1, const double *vz2, const double *vz3, double *value_dz,
                      const safara_dims3_t *dims, double h, void *stream) {
    int dev;
    int rc = current_device(&dev);
    if (rc) return rc;
    if (!dims || !vz1 || !vz2 || !vz3 || !value_dz) return SAFARA_ERR_ARG;
    if (!(h != 0.0) || h - h != 0.0) return SAFARA_ERR_ARG;  // zero, NaN or infinite
    const safara_dims3_t &d = *dims;
    if (d.nx < 2 || d.ny < 2 || d.nz < 2) return SAFARA_ERR_SHAPE;
    if (d.sy < d.nx || d.sk < (long long)d.sy * d.ny) return SAFARA_ERR_LAYOUT;
    const long long maxo = (long long)(d.nx - 1) + (long long)d.sy * (d.ny - 1) +
                           (long long)d.sk * (d.nz - 1);
    if (maxo >= (1LL << 31)) return SAFARA_ERR_TOO_LARGE;  // `small`
    if (((uintptr_t)vz1 | (uintptr_t)vz2 | (uintptr_t)vz3 | (uintptr_t)value_dz) & 7u)
        return SAFARA_ERR_ALIGN;
    const long long bytes = (maxo + 1) * (long long)sizeof(double);
    if (overlaps(value_dz, bytes, vz1, bytes) || overlaps(value_dz, bytes, vz2, bytes) ||
        overlaps(value_dz, bytes, vz3, bytes))
        return SAFARA_ERR_ARG;
    cudaError_t e = launch_seismic_dz(vz1, vz2, vz3, value_dz, d.nx, d.ny, d.nz, d.sy, d.sk, h,
                                      g_dev[dev].sms, (cudaStream_t)stream);
    if (e != cudaSuccess) return SAFARA_ERR_CUDA;
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return SAFARA_OK;
}

int64_t safara_launch_count(void) { return g_launches.load(); }

int safara_kernel_info(int which, safara_kernel_info_t *out) {
    if (!out || (which != 0 && which != 1)) return SAFARA_ERR_ARG;
    int dev;
    int rc = current_device(&dev);
    if (rc) return rc;
    const DeviceState &st = g_dev[dev];
    if (g_tune.ws) {
        // the warp-specialised kernel (one-segment lockstep launches, e.g.
        // every full-grid pass at class C): NAS coefficients instantiation
        const cudaFuncAttributes *a = which ? st.attr_ws_strict : st.attr_ws_fast;
        out->regs_per_thread = a[0].numRegs;  // launch allocation (setmaxnreg moves them)
        out->local_bytes = (int)a[0].localSizeBytes;
        out->smem_bytes = (int)(a[0].sharedSizeBytes + WS_SMEM_BYTES);
        out->threads_per_cta = WS_THREADS;
        out->ctas_per_sm = 1;
        out->tile_x = TX;
        out->tile_y = TY;
        out->stages = WS_US;
        return SAFARA_OK;
    }
    const cudaFuncAttributes *a = which ? st.attr_strict : st.attr_fast;
    out->regs_per_thread = a[0].numRegs;
    // local (spill) bytes of the production instantiation (NAS coefficients,
    // no aux); the general / aux instantiations spill 4-8 B in their segment
    // setup, outside the k march (profiles/ptxas_r01.txt)
    out->local_bytes = (int)a[0].localSizeBytes;
    out->smem_bytes = (int)(a[0].sharedSizeBytes + SMEM_BYTES);
    out->threads_per_cta = NTHREADS;
    out->ctas_per_sm = which ? st.ctas_strict : st.ctas_fast;
    out->tile_x = TX;
    out->tile_y = TY;
    out->stages = STAGES;
    return SAFARA_OK;
}

const char *safara_strerror(int code) {
    switch (code) {
        case SAFARA_OK: return "success";
        case SAFARA_ERR_ARG: return "invalid argument (null pointer, aliasing or bad flag)";
        case SAFARA_ERR_SHAPE: return "invalid shape (extent < 6, slab < 2 planes or bad k range)";
        case SAFARA_ERR_LAYOUT: return "invalid layout (strides overlap, sy < nx or j not second-fastest)";
        case SAFARA_ERR_ALIGN: return "misaligned pointer or stride (16-byte TMA rule)";
        case SAFARA_ERR_TOO_LARGE: return "largest offset >= 2^31: the `small` (32-bit offset) claim is false";
        case SAFARA_ERR_NOT_INIT: return "safara_rhs_init was not called for the current device";
        case SAFARA_ERR_CUDA: return "CUDA runtime or driver error";
        case SAFARA_ERR_NO_DEVICE: return "no sm_100 device at this index";
        case SAFARA_ERR_NCCL: return "NCCL error (library not loadable, communicator or P2P failure)";
        default: return "unknown error code";
    }
}

}  // extern "C"
