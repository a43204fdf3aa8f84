// rhs_ws.cuh -- warp-specialised variant of the compute_rhs pass (round 2).
//
// Same arithmetic and the same per-thread k march as rhs_kernel.cuh (one
// thread per (i,j) column, register window along k = SAFARA's
// inter-iteration scalar replacement, Fig. 6),
// but the CTA is split into two roles:
//
//  * 4 PRODUCER warps (one warpgroup, registers handed to the consumers with
//    setmaxnreg.dec): one lane issues the TMA loads of the u / forcing plane
//    tiles into the STAGES-deep ring when the consumers release a slot
//    (mbarrier `empty`, no atomics); then all 128 producer threads evaluate
//    the step-0 fields rho_i = 1/u1 and square (App. A step 0) ONCE for every
//    point of the plane tile plus a halo of one, into an aux ring in shared
//    memory, and signal `afull`.
//  * TY CONSUMER warps (setmaxnreg.inc), one tile row each: every neighbour's
//    rho_i / square now comes from that aux tile (one 16-byte load) instead of
//    being recomputed per use (round 1 evaluated aux_of four times per point:
//    own, the xi tile-edge lanes, both eta rows) or shuffled; the own values
//    of plane k+1 are loaded, not computed.
//
// SAFARA's cost model (L x C) placed the values
// with reuse > 1 that other threads need in shared memory; the aux fields have
// reuse 5 (own + 4 in-plane neighbours) and were recomputed in round 1 only
// because a consumer-side producer needed cross-warp waits.  A producer
// warpgroup working ahead of the consumers removes those waits.
//
// Scope: launches whose CTAs each own ONE (column tile, k range) segment
// (the lockstep schedule) without the f1 aux output or the f2 peer halo;
// everything else runs rhs_kernel.cuh (launch() decides).
#pragma once

namespace safara {
namespace dev {

#ifndef SAFARA_WS_XOREG
#define SAFARA_WS_XOREG 1  // edge-tile xi case bits in a register (0: recomputed per step, A/B: 4 % slower)
#endif
#ifndef SAFARA_WS_SLEEP
#define SAFARA_WS_SLEEP 20000   // producer waits: suspend-time hint (ns), 0 = plain try_wait
#endif
__device__ __forceinline__ void ws_pwait(uint64_t *bar, uint32_t parity) {
#if SAFARA_WS_SLEEP > 0
    mbar_wait_sleep(bar, parity, SAFARA_WS_SLEEP);
#else
    mbar_wait(bar, parity);
#endif
}
#ifndef SAFARA_WS_PROBE
#define SAFARA_WS_PROBE 0  // timing probes (wrong rhs): 1 no zeta dissipation, 2 no xi dissipation (mid tiles)
#endif
#ifndef SAFARA_WS_NORM_PROBE
#define SAFARA_WS_NORM_PROBE 0  // timing probe: the fused norm without its in-loop accumulation (wrong norm)
#endif
#ifndef SAFARA_WS_LATE_FULL
#define SAFARA_WS_LATE_FULL 1  // wait for plane k+2's tile just before its own-column read (A/B: -0.6 %, profiles/ab_late_placement_r02s2.txt)
#endif
#ifndef SAFARA_WS_FORCING_LAST
#define SAFARA_WS_FORCING_LAST 0  // production: add forcing at the end of the step
#endif
#ifndef SAFARA_WS_CSLEEP
#define SAFARA_WS_CSLEEP 0      // consumer waits: suspend-time hint (ns), 0 = plain try_wait spin
#endif
#ifndef SAFARA_WS_STORE
#define SAFARA_WS_STORE 0       // rhs stores: 0 st.global.cs, 1 default policy
#endif
__device__ __forceinline__ void ws_cwait(uint64_t *bar, uint32_t parity) {
#if SAFARA_WS_CSLEEP > 0
    mbar_wait_sleep(bar, parity, SAFARA_WS_CSLEEP);
#else
    mbar_wait(bar, parity);
#endif
}
__device__ __forceinline__ double *ws_u() { return reinterpret_cast<double *>(smem_raw); }
__device__ __forceinline__ double2 *ws_aux() {
    return reinterpret_cast<double2 *>(smem_raw + WS_U_BYTES);
}
__device__ __forceinline__ double *ws_f() {
    return reinterpret_cast<double *>(smem_raw + WS_U_BYTES + WS_AUX_BYTES);
}
__device__ __forceinline__ uint64_t *ws_full() {
    return reinterpret_cast<uint64_t *>(smem_raw + WS_BAR_OFF);
}
__device__ __forceinline__ uint64_t *ws_afull() { return ws_full() + WS_US; }
__device__ __forceinline__ uint64_t *ws_empty() { return ws_full() + 2 * WS_US; }
__device__ __forceinline__ uint64_t *ws_ffull() { return ws_full() + 3 * WS_US; }
__device__ __forceinline__ uint64_t *ws_fempty() { return ws_ffull() + WS_FS; }

// TMA of u plane k (tile with halo 2) into u slot `slot`, of forcing plane k
// into forcing slot `slot` (coordinates as rhs_kernel.cuh issue_plane).
__device__ __forceinline__ void ws_issue_u(const CUtensorMap *umap, const Params &P, int i0,
                                           int j0, int k, int slot) {
    const int kb = k - P.k0 + P.ukoff, jc = j0 - 2;
    const int c1 = P.pos_j == 1 ? jc : (P.pos_m == 1 ? 0 : kb);
    const int c2 = P.pos_j == 2 ? jc : (P.pos_m == 2 ? 0 : kb);
    const int c3 = P.pos_j == 3 ? jc : (P.pos_m == 3 ? 0 : kb);
    uint64_t *bar = &ws_full()[slot];
    if (k >= P.pk_hi) {  // f2: a neighbour's plane (own column read by peer_col)
        mbar_arrive(bar);
        return;
    }
    mbar_expect_tx(bar, TMA_BYTES);
    tma_load_4d(ws_u() + (size_t)slot * U_SLOT, umap, bar, i0 - HX, c1, c2, c3);
}
__device__ __forceinline__ void ws_issue_f(const CUtensorMap *fmap, const Params &P, int i0,
                                           int j0, int k, int slot) {
    const int kf = k - P.k0;
    const int f1 = P.pos_j == 1 ? j0 : (P.pos_m == 1 ? 0 : kf);
    const int f2 = P.pos_j == 2 ? j0 : (P.pos_m == 2 ? 0 : kf);
    const int f3 = P.pos_j == 3 ? j0 : (P.pos_m == 3 ? 0 : kf);
    uint64_t *bar = &ws_ffull()[slot];
    mbar_expect_tx(bar, TMA_BYTES_F);
    tma_load_4d(ws_f() + (size_t)slot * F_SLOT, fmap, bar, i0 - 1, f1, f2, f3);
}

__device__ __forceinline__ void setmaxnreg_inc_consumer() {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;\n" ::"n"(WS_CREG));
}
__device__ __forceinline__ void setmaxnreg_dec_producer() {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;\n" ::"n"(SAFARA_WS_PREG));
}

// The CTA's segment in the lockstep schedule: column tile `col`, global
// planes [ka, kb).
__device__ __forceinline__ void ws_segment(const Params &P, int &col, int &ka, int &kb) {
    const int c = (int)blockIdx.x;
    col = c % P.ncol;
    const int part = c / P.ncol;
    const int np = P.nplanes + P.split_bias;
    const int b0 = max(0, min((part * np) / P.parts, P.nplanes));
    const int b1 = part + 1 == P.parts ? P.nplanes : max(0, min(((part + 1) * np) / P.parts, P.nplanes));
    ka = P.ka0 + b0;
    kb = P.ka0 + b1;
}

// Producer warpgroup.  Warp TY: one lane issues the TMA loads -- planes 0..
// STAGES-1 up front, then plane s+STAGES as soon as the consumers release
// plane s (`empty`); it never waits for anything else, so a refill is never
// held up behind aux work.  Warps TY+1..TY+3 (96 threads): for every plane,
// once its tile has landed (`full`), rho_i / square of the tile + halo 1 into
// the aux ring, then `afull` (count WS_AW).
constexpr int WS_AW = WS_PW - 1;  // aux warps
__device__ __forceinline__ void ws_producer(const CUtensorMap *umap, const CUtensorMap *fmap,
                                            const Params &P) {
    int col, ka, kb;
    ws_segment(P, col, ka, kb);
    if (ka >= kb) return;
    const int i0 = 1 + (col % P.ntx) * TX, j0 = 1 + (col / P.ntx) * TY;
    const int nu = kb - ka + 2;  // u planes ka .. kb+1
    const int nf = kb - ka;      // forcing planes ka .. kb-1
    const int warp = (int)threadIdx.x / 32, lane = (int)threadIdx.x % 32;
    uint64_t *full = ws_full(), *afull = ws_afull();
    if (warp == TY) {
        if (lane != 0) return;  // (the norm epilogue is entered by rhs_body_ws)
        // in deadline order: step t reads u(t+2) (own column) and f(t)
        for (int s = 0; s < WS_US && s < nu; ++s) ws_issue_u(umap, P, i0, j0, ka + s, s);
        for (int s = 0; s < WS_FS && s < nf; ++s) ws_issue_f(fmap, P, i0, j0, ka + s, s);
        for (int t = 0;; ++t) {
            const int su_ = t + 2 + (WS_US - 2), sf = t + WS_FS;  // next u / f to issue
            const bool mu = su_ < nu, mf = sf < nf;
            if (!mu && !mf) break;
            // step t releases forcing(t) at its start and u(t) after its
            // eta stencil: refill in that order
            if (mf) {  // f(sf) reuses the slot of f(sf - WS_FS), released at step sf - WS_FS
                const int r = sf - WS_FS;
                ws_pwait(&ws_fempty()[r % WS_FS], (uint32_t)(r / WS_FS) & 1u);
                ws_issue_f(fmap, P, i0, j0, ka + sf, sf % WS_FS);
            }
            if (mu) {  // u(su_) reuses the slot of u(su_ - WS_US), released at step su_ - WS_US
                const int r = su_ - WS_US;
                ws_pwait(&ws_empty()[r % WS_US], (uint32_t)(r / WS_US) & 1u);
                ws_issue_u(umap, P, i0, j0, ka + su_, su_ % WS_US);
            }
        }
        return;
    }
    const int pt = (int)threadIdx.x - (TY + 1) * 32;  // 0 .. 32*WS_AW-1
    double2 *ax = ws_aux();
    for (int s = 0; s < nu; ++s) {
        const int slot = s % WS_US;
        ws_pwait(&full[slot], (uint32_t)(s / WS_US) & 1u);
        // rho_i, square of every point of the tile + halo 1 (App. A step 0);
        // none for a neighbour's plane (f2: no tile was loaded)
        const double *ut = ws_u() + (size_t)slot * U_SLOT;
        double2 *at = ax + (size_t)slot * A_SLOT;
        for (int p = ka + s < P.pk_hi ? pt : A_SLOT; p < A_SLOT; p += WS_AW * 32) {
            const int r = p / AXW, c = p - r * AXW;
            const int ui = (r + 1) * UX + (c + HX - 1);
            double rho, sq;
            aux_of(ut[ui], ut[ui + UPM], ut[ui + 2 * UPM], ut[ui + 3 * UPM], rho, sq);
            at[p] = make_double2(rho, sq);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&afull[slot]);  // release: the aux stores above
    }
}

// Consumer per-thread state (as rhs_kernel.cuh Seg, aux from smem).
struct SegW {
    double *rptr;
    int uc, ac;
    bool active, mid_x;
    int fidx;        // i-face copy (P.iface_tiles): forcing-tile index of this lane's value, or -1
    double *fptr;    //   and its rhs address at the current plane
    int ycase;
#if SAFARA_WS_XOREG
    int xo;
#endif
    double a[3][5];
    int colo;        // f2 (PEER): own column offset i + sy*j for the neighbours' planes
    double rq, sq;   // rho_i / square of plane k-1 (planes k, k+1: from the aux ring)
    double tp[5];
    double ss[5];    // NORM: this thread's sum of rhs_m^2 over its march (f1)
};

// Edge column tiles: the xi-dissipation case bits and i+-2 redirections of
// this lane (rhs_kernel.cuh SAFARA_XREG), from blockIdx / laneid.
__device__ __forceinline__ int ws_xo(const Params &P) {
    const int col = (int)blockIdx.x % P.ncol;
    const int i = 1 + (col % P.ntx) * TX + (int)(threadIdx.x % 32);
    const Cases cs = cases_of(i, P.nx);
    return (i == P.nx - 3 ? 3 : 2) | ((i == 2 ? 3 : 2) << 8) | (cs.hm1 ? 1 << 16 : 0) |
           (cs.five ? 1 << 17 : 0) | (cs.hp1 ? 1 << 18 : 0);
}

// FAST steps (interior planes: k and k+1 take the mid zeta cases, no peer
// plane involved): every wait at the top and then ONE branch-free basic
// block -- xi dissipation in the per-lane table form for every tile, eta in
// a per-warp coefficient form for every row, predicated stores -- so the
// scheduler can overlap the shared-memory loads of all three directions with
// the FP64 work (the generic step is ~8 basic blocks, several of them "load,
// then use at once").  Bitwise identical to the generic step (see
// diss_eta_coef).
#ifndef SAFARA_WS_FAST
#define SAFARA_WS_FAST 0  // A/B on B200: 1 % slower (profiles/ab_fast_r02.txt)
#endif
// eta dissipation weights {c-2, c-1, c0, c+1, c+2} of the NAS cases
// (0 interior, 1 j=1, 2 j=2, 3 j=ny-3, 4 j=ny-2): t = c-2*a-2, then
// fma(c-1, a-1, t), + c0*a0, fma(c+1, a+1, t), fma(c+2, a+2, t).  A zero
// weight multiplies a finite value (exact 0 / t + 0 = t) and unit / -4 / 6 /
// 5 products are the NAS ones, so every case rounds exactly as the NAS text
// (diss_terms_case) in STRICT; the production build contracts the same way
// as the interior form.
__constant__ double c_eta_coef[5][5] = {{1.0, -4.0, 6.0, -4.0, 1.0},
                                         {0.0, 0.0, 5.0, -4.0, 1.0},
                                         {0.0, -4.0, 6.0, -4.0, 1.0},
                                         {1.0, -4.0, 6.0, -4.0, 0.0},
                                         {1.0, -4.0, 5.0, 0.0, 0.0}};
__device__ __forceinline__ void diss_eta_coef(double (&t)[5], const double (&am2)[5],
                                              const double (&am1)[5], const double (&a0)[5],
                                              const double (&ap1)[5], const double (&ap2)[5],
                                              const double *ce) {
    const double cm2 = ce[0], cm1 = ce[1], cc = ce[2], cp1 = ce[3], cp2 = ce[4];
#pragma unroll
    for (int m = 0; m < 5; ++m) {
        double x = cm2 * am2[m];
        x = __fma_rn(cm1, am1[m], x);
        x = x + cc * a0[m];
        x = __fma_rn(cp1, ap1[m], x);
        t[m] = __fma_rn(cp2, ap2[m], x);
    }
}
__device__ __forceinline__ void st_cs_pred(double *p, double v, bool pred) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q st.global.cs.f64 [%0], %1;\n\t}" ::"l"(p),
                 "d"(v), "r"((unsigned)pred)
                 : "memory");
}

template <int R, bool UD, bool AUX, bool NORM, bool PEER, bool FAST = false>
__device__ __forceinline__ void ws_step(SegW &g, const Params &P, int k, int q, int ka) {
    constexpr int Q = R % 3, Z = (R + 1) % 3, PI = (R + 2) % 3;  // planes k-1, k, k+1
    const Coef &C = P.c;
    double *const su = ws_u();
    const double2 *const ax = ws_aux();
    const double *s = su + (size_t)(q % WS_US) * U_SLOT;
    const double2 *a0 = ax + (size_t)(q % WS_US) * A_SLOT;
    double acc[5];
    if (FAST) {  // every wait of the step first
        ws_cwait(&ws_ffull()[q % WS_FS], (uint32_t)(q / WS_FS) & 1u);
        ws_cwait(&ws_afull()[(q + 1) % WS_US], (uint32_t)((q + 1) / WS_US) & 1u);
        ws_cwait(&ws_full()[(q + 2) % WS_US], (uint32_t)((q + 2) / WS_US) & 1u);
    }
    // forcing(k): its own ring, released right after this read.  FLAST
    // (production, zeta first): the step starts from the zeta partial sum and
    // adds forcing at its end, so the forcing wait leaves the top of the step
    // (the sum of the formed terms re-associated: reading c6)
    constexpr bool FLAST = SAFARA_WS_FORCING_LAST && SAFARA_ZETA_FIRST && !SAFARA_STRICT_BUILD &&
                           !FAST;
    auto read_forcing = [&](double (&f)[5]) {
        if (!FAST) ws_cwait(&ws_ffull()[q % WS_FS], (uint32_t)(q / WS_FS) & 1u);
        const double *fs = ws_f() + (size_t)(q % WS_FS) * F_SLOT;
        // own forcing: (ty, tx+1) of the FX-wide tile = aux-tile index - AXW
        static_assert(FX == AXW, "forcing and aux tiles share the row width");
#pragma unroll
        for (int m = 0; m < 5; ++m) f[m] = fs[m * TY * FX - AXW + g.ac];
        if (g.fidx >= 0) {  // one i-face value of this row: rhs = forcing (reading c3)
            __stcs(g.fptr, fs[g.fidx]);
            g.fptr += SK(r);
        }
        __syncwarp();
        if ((threadIdx.x & 31) == 0) mbar_arrive(&ws_fempty()[q % WS_FS]);
    };
    if (!FLAST) read_forcing(acc);
    // the aux of plane k+1 (own rho_i / square for the zeta flux) is in place
    // and plane k+2's tile has landed (own column read at the end of the
    // step); plane k+2's aux is not needed yet, so its evaluation overlaps
    // this step
    if (!FAST) {
        // zeta last: the aux of plane k+1 is first needed by zeta (below)
        if (SAFARA_ZETA_FIRST) ws_cwait(&ws_afull()[(q + 1) % WS_US], (uint32_t)((q + 1) / WS_US) & 1u);
#if !SAFARA_WS_LATE_FULL
        ws_cwait(&ws_full()[(q + 2) % WS_US], (uint32_t)((q + 2) / WS_US) & 1u);
#endif
    }
    const double *const s2 = su + (size_t)((q + 2) % WS_US) * U_SLOT;
    double an[5];
    const double (&wz)[5] = g.a[Z];
    const double2 own = a0[g.ac];  // rho_i / square of plane k
    const double r0 = own.x, s0 = own.y;
    double vc[3];
    vc[0] = wz[1] * r0;
    vc[1] = wz[2] * r0;
    vc[2] = wz[3] * r0;
    const double qsc = s0 * r0;
    const double pc = wz[4] * r0;
    if (AUX && g.active) {  // f1: the step-0 fields of this point (plane k)
        const int kl = k - P.k0;
        const int off = (int)(g.rptr - P.r) - SK(r) * kl;
        store_aux(P, off, kl, r0, vc[0], vc[1], vc[2], s0, qsc, wz[4]);
    }
    auto zeta = [&]() {
        Nb p, qn;
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            p.u[m] = g.a[PI][m];
            qn.u[m] = g.a[Q][m];
        }
        if (PEER && !FAST && k + 1 >= P.pk_hi) {  // f2: plane k+1 is the upper neighbour's
            aux_of(p.u[0], p.u[1], p.u[2], p.u[3], p.rho, p.sq);
        } else {
            const double2 o1 = ax[(size_t)((q + 1) % WS_US) * A_SLOT + g.ac];  // plane k+1
            p.rho = o1.x; p.sq = o1.y;
        }
        qn.rho = g.rq; qn.sq = g.sq;
        flux_dir<3, FLAST, UD>(acc, wz, vc, qsc, pc, p, qn, C, 2);
    };
#if SAFARA_ZETA_FIRST
    zeta();
#endif
    {   // xi: neighbours' rho_i / square from the aux tile
        Nb p, qn;
        load5(p.u, s, g.uc + 1);
        load5(qn.u, s, g.uc - 1);
        const double2 ap = a0[g.ac + 1], aq = a0[g.ac - 1];
        p.rho = ap.x; p.sq = ap.y;
        qn.rho = aq.x; qn.sq = aq.y;
        double t[5];
        {
            double pp[5], qq[5];
            if (FAST) {  // the table form for every tile (mid tiles: offsets 2, weights -4/6/-4)
                const int xo = g.xo;
                load5(pp, s, g.uc + (xo & 0xff));
                load5(qq, s, g.uc - ((xo >> 8) & 0xff));
                diss_terms_table(t, qq, qn.u, wz, p.u, pp, (xo & (1 << 16)) ? -4.0 : 0.0,
                                 (xo & (1 << 17)) ? 5.0 : 6.0, (xo & (1 << 18)) ? -4.0 : 0.0);
            } else if (g.mid_x) {
#if SAFARA_WS_PROBE == 2  // timing probe: no xi dissipation loads / terms (wrong rhs)
#pragma unroll
                for (int m = 0; m < 5; ++m) t[m] = 0.0;
#else
                load5(pp, s, g.uc + 2);
                load5(qq, s, g.uc - 2);
                diss_terms<false>(t, qq, qn.u, wz, p.u, pp, Cases{});
#endif
            } else {
#if SAFARA_WS_XOREG
                const int xo = g.xo;
#else
                const int xo = ws_xo(P);  // edge tiles only: recomputed, no live register
#endif
                load5(pp, s, g.uc + (xo & 0xff));
                load5(qq, s, g.uc - ((xo >> 8) & 0xff));
                diss_terms_table(t, qq, qn.u, wz, p.u, pp, (xo & (1 << 16)) ? -4.0 : 0.0,
                                 (xo & (1 << 17)) ? 5.0 : 6.0, (xo & (1 << 18)) ? -4.0 : 0.0);
            }
        }
        flux_dir<1, false, UD>(acc, wz, vc, qsc, pc, p, qn, C, 0);
#if SAFARA_WS_PROBE != 2
        diss_apply(acc, t, C.dssp);
#endif
    }
    {   // eta
        Nb p, qn;
        load5(p.u, s, g.uc + UX);
        load5(qn.u, s, g.uc - UX);
        const double2 ap = a0[g.ac + AXW], aq = a0[g.ac - AXW];
        p.rho = ap.x; p.sq = ap.y;
        qn.rho = aq.x; qn.sq = aq.y;
        double t[5];
        {
            double pp[5], qq[5];
            load5(pp, s, g.uc + 2 * UX);
            load5(qq, s, g.uc - 2 * UX);
            if (FAST)
                diss_eta_coef(t, qq, qn.u, wz, p.u, pp, c_eta_coef[g.ycase]);
            else
                diss_terms_case(t, qq, qn.u, wz, p.u, pp, g.ycase);
        }
        // every read of plane k's slot (u, forcing, aux) is done: release it
        __syncwarp();
        if ((threadIdx.x & 31) == 0) mbar_arrive(&ws_empty()[q % WS_US]);
        flux_dir<2, false, UD>(acc, wz, vc, qsc, pc, p, qn, C, 1);
        diss_apply(acc, t, C.dssp);
    }
#if !SAFARA_ZETA_FIRST
    if (!FAST) ws_cwait(&ws_afull()[(q + 1) % WS_US], (uint32_t)((q + 1) / WS_US) & 1u);
    zeta();
#endif
#if SAFARA_WS_LATE_FULL
    // plane k+2's tile is read only here (own column): wait for it here, so
    // the first step of a pass computes plane k's xi/eta/zeta while plane
    // k+2 is still arriving (the ring-fill latency of short slab passes)
    if (!FAST) ws_cwait(&ws_full()[(q + 2) % WS_US], (uint32_t)((q + 2) / WS_US) & 1u);
#endif
    if (PEER && !FAST && k + 2 >= P.pk_hi)
        peer_col(an, P, k + 2, g.colo);  // f2: the upper neighbour's own column
    else
        load5(an, s2, g.uc);
#if SAFARA_WS_PROBE != 1  // 1: timing probe without the zeta dissipation (wrong rhs)
    {
        double t_z[5];
        if (FAST || is_mid(k, P.nz)) {
#pragma unroll
            for (int m = 0; m < 5; ++m) t_z[m] = __fma_rn(-4.0, g.a[PI][m], g.tp[m]) + an[m];
        } else {
            const Cases c = cases_of(k, P.nz);
#pragma unroll
            for (int m = 0; m < 5; ++m) {
                const double y1 = c.hp1 ? g.a[PI][m] : 0.0;
                const double y2 = c.hp2 ? an[m] : 0.0;
                t_z[m] = __fma_rn(-4.0, y1, g.tp[m]) + y2;
            }
        }
        diss_apply(acc, t_z, C.dssp);
    }
#endif
    if (FLAST) {
        double fv[5];
        read_forcing(fv);
#pragma unroll
        for (int m = 0; m < 5; ++m) acc[m] = acc[m] + fv[m];
    }
    if (FAST) {  // predicated stores: no branch
        double *rp = g.rptr;
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            const double v = acc[m] * C.dt;
            st_cs_pred(rp, v, g.active);
            if (NORM) {
                const double va = g.active ? v : 0.0;
                g.ss[m] = __fma_rn(va, va, g.ss[m]);
            }
            rp += SM(r);
        }
    } else if (g.active) {
        double *rp = g.rptr;
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            const double v = acc[m] * C.dt;
#if SAFARA_WS_STORE == 0
            __stcs(rp, v);
#else
            *rp = v;
#endif
            if (NORM && !SAFARA_WS_NORM_PROBE) g.ss[m] = __fma_rn(v, v, g.ss[m]);  // f1: NPB rhs_norm numerator
            rp += SM(r);
        }
    }
    g.rptr += SK(r);
#if SAFARA_WS_PROBE != 1
    zeta_partial(g.tp, g.a[Q], g.a[Z], g.a[PI], k + 1, P.nz, FAST || is_mid(k + 1, P.nz));
#endif
#pragma unroll
    for (int m = 0; m < 5; ++m) g.a[Q][m] = an[m];
    g.rq = r0;  // plane k is plane k-1 of the next step
    g.sq = s0;
    (void)ka;
}

// f1 fused rhs_norm, after the march.  Consumers: warp trees of their
// per-thread sums into red[warp][m], then arrive on named barrier 2.  The
// producer warpgroup (idle by then, few registers -- so the consumers' k march
// keeps its allocation) waits there, forms this CTA's partials (warps in
// order: deterministic for a given launch) and the last CTA to finish sums
// every CTA's partials in CTA order and finishes NPB rhs_norm (no second
// launch), leaving the counter at 0.
__shared__ double ws_red[TY][5];
__shared__ int ws_last;
constexpr int WS_NRED = 25;  // last-CTA reduction: threads per component
__shared__ double ws_red2[5][WS_NRED];
constexpr int WS_NORM_BAR = 2;

__device__ __forceinline__ void ws_norm_consumer(const double (&ss)[5], int tid) {
    const int warp = tid / 32, lane = tid % 32;
#pragma unroll
    for (int m = 0; m < 5; ++m) {
        double v = ss[m];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
        if (lane == 0) ws_red[warp][m] = v;
    }
    asm volatile("bar.arrive %0, %1;" ::"n"(WS_NORM_BAR), "n"(WS_THREADS) : "memory");
}

__device__ __forceinline__ void ws_norm_producer(const Params &P) {
    asm volatile("bar.sync %0, %1;" ::"n"(WS_NORM_BAR), "n"(WS_THREADS) : "memory");
    const int pt = (int)threadIdx.x - TY * 32;  // 0 .. 127
    if (pt < 5) {
        double t = 0.0;
        for (int w = 0; w < TY; ++w) t += ws_red[w][pt];
        P.norm_part[pt * P.ncta + (int)blockIdx.x] = t;
    }
    asm volatile("bar.sync 3, 128;" ::: "memory");  // producers: partials stored
    if (pt == 0) {
        // one acq_rel atomic instead of fence + atomic: releases this CTA's
        // partials (ordered before it by the barrier; release is cumulative)
        // and, for the last CTA, acquires every other CTA's
        unsigned long long old;
        asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], 1;"
                     : "=l"(old) : "l"(P.norm_ctr) : "memory");
        ws_last = old == (unsigned long long)P.ncta - 1;
    }
    asm volatile("bar.sync 3, 128;" ::: "memory");
    if (ws_last) {
        // the last CTA: 125 threads sum the CTA partials of component
        // pt / 25 strided by 25 (fixed order, loads independent), then 5
        // threads add the 25 sums in order -- deterministic for a given grid,
        // and ~2 dependent L2 round trips instead of ncta (the partials
        // were acquired by thread 0's atomic; the barrier orders the loads)
        if (pt < 5 * WS_NRED) {
            const int m = pt / WS_NRED, s0 = pt - m * WS_NRED;
            const double *part = P.norm_part + m * P.ncta;
            double t = 0.0;
#pragma unroll 8
            for (int b = s0; b < P.ncta; b += WS_NRED) t += __ldcg(part + b);
            ws_red2[m][s0] = t;
        }
        asm volatile("bar.sync 3, 128;" ::: "memory");
        if (pt < 5) {
            double t = 0.0;
#pragma unroll
            for (int s = 0; s < WS_NRED; ++s) t += ws_red2[pt][s];
            P.norm_out[pt] = P.norm_npts > 0.0 ? sqrt(t / P.norm_npts) : t;
        }
        if (pt == 0) *P.norm_ctr = 0ull;
    }
}

template <bool UD, bool AUX, bool NORM, bool PEER>
__device__ __forceinline__ void ws_consumer(const Params &P) {
    int col, ka, kb;
    ws_segment(P, col, ka, kb);
    const int tid = (int)threadIdx.x;
    if (ka >= kb) {
        if (NORM) {  // an empty k-part still reports (zero) to the norm barrier
            const double z[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
            ws_norm_consumer(z, tid);
        }
        return;
    }
    const int tx = tid % TX, ty = tid / TX;
    const int i0 = 1 + (col % P.ntx) * TX, j0 = 1 + (col / P.ntx) * TY;
    const int i = i0 + tx, j = j0 + ty;
    const int nx_s = reread(P.nx), ny_s = reread(P.ny);
    SegW g;
    g.active = (i <= nx_s - 2) && (j <= ny_s - 2);
    // the i-face columns (P.iface_tiles): in the first column tile lanes 0..4
    // copy component `lane` of rhs(0, j, k) = forcing(0, j, k), in the last
    // column tile lanes 5..9 that of i = nx-1 (rows 1..ny-2); the forcing
    // tile's columns i0-1 .. i0+TX hold both, so each warp adds one shared
    // load and one store per step (5 lanes active)
    g.fidx = -1;
    g.fptr = nullptr;
    if (!AUX && P.iface_tiles && j <= ny_s - 2) {
        const int ctile = (col % P.ntx);
        int fi = -1, m = -1;
        if (tx < 5 && ctile == 0) { fi = 0; m = tx; }
        else if (tx >= 5 && tx < 10 && ctile == P.ntx - 1) { fi = nx_s - 1; m = tx - 5; }
        if (fi >= 0) {
            g.fidx = m * TY * FX + ty * FX + (fi - (i0 - 1));
            g.fptr = P.r + ((idx_t)fi + SY(r) * j + SM(r) * m + SK(r) * (ka - P.k0));
        }
    }
    g.uc = (ty + 2) * UX + (tx + HX);
    g.ac = (ty + 1) * AXW + (tx + 1);
    g.mid_x = is_mid(i0, P.nx) && is_mid(i0 + TX - 1, P.nx);
    g.ycase = is_mid(j, ny_s) ? 0 : j == 1 ? 1 : j == 2 ? 2 : j == ny_s - 3 ? 3 : 4;
#if SAFARA_WS_XOREG
    g.xo = ws_xo(P);
#endif
    g.rptr = P.r + ((idx_t)i + SY(r) * j + SK(r) * (ka - P.k0));
    double *su = ws_u();
    {   // window: planes ka-2, ka-1 from global memory, ka and ka+1 from the ring
        const int ic = min(i, nx_s - 1), jc = min(j, ny_s - 1);
        const int lk = ka - P.k0 + P.ukoff;
        const double *uc0 = P.u + (idx_t)(ic + SY(u) * jc);
        const int colo = ic + P.sy * jc;
        g.colo = colo;
        if (ka - 1 < P.pk_lo) {  // f2: planes below the slab are the lower neighbour's
            peer_col(g.a[0], P, ka - 1, colo);
        } else {
#pragma unroll
            for (int m = 0; m < 5; ++m)
                g.a[0][m] = lk - 1 >= 0 ? __ldg(uc0 + SM(u) * m + SK(u) * (lk - 1)) : 0.0;
        }
        double am2[5];
        if (ka - 2 < P.pk_lo) {
            peer_col(am2, P, ka - 2, colo);
        } else {
#pragma unroll
            for (int m = 0; m < 5; ++m)
                am2[m] = lk - 2 >= 0 ? __ldg(uc0 + SM(u) * m + SK(u) * (lk - 2)) : 0.0;
        }
        aux_of(g.a[0][0], g.a[0][1], g.a[0][2], g.a[0][3], g.rq, g.sq);
        mbar_wait(&ws_afull()[0], 0u);
        load5(g.a[1], su, g.uc);
        zeta_partial(g.tp, am2, g.a[0], g.a[1], ka, P.nz, is_mid(ka, P.nz));
        mbar_wait(&ws_full()[1], 0u);
        if (PEER && ka + 1 >= P.pk_hi)
            peer_col(g.a[2], P, ka + 1, colo);
        else
            load5(g.a[2], su + (size_t)1 * U_SLOT, g.uc);
    }
#pragma unroll
    for (int m = 0; m < 5; ++m) g.ss[m] = 0.0;
    int k = ka, q = 0;
#if SAFARA_WS_FAST
    // planes whose step can run FAST: k and k+1 interior in zeta and plane
    // k+2 local (f2); CTA-uniform, so one uniform branch per step
    const int kf_lo = 3, kf_hi = min(P.nz - 5, PEER ? P.pk_hi - 3 : P.nz);
#define WS_STEP(RR, KK, QQ)                                                  \
    if ((KK) >= kf_lo && (KK) <= kf_hi)                                      \
        ws_step<RR, UD, AUX, NORM, PEER, true>(g, P, KK, QQ, ka);           \
    else                                                                     \
        ws_step<RR, UD, AUX, NORM, PEER, false>(g, P, KK, QQ, ka);
#else
#define WS_STEP(RR, KK, QQ) ws_step<RR, UD, AUX, NORM, PEER, false>(g, P, KK, QQ, ka);
#endif
#pragma unroll 1
    for (; k + 3 <= kb; k += 3, q += 3) {
        WS_STEP(0, k, q)
        WS_STEP(1, k + 1, q + 1)
        WS_STEP(2, k + 2, q + 2)
    }
#undef WS_STEP
    if (k < kb) {
        ws_step<0, UD, AUX, NORM, PEER>(g, P, k, q, ka);
        if (k + 1 < kb) ws_step<1, UD, AUX, NORM, PEER>(g, P, k + 1, q + 1, ka);
    }
    if (NORM) ws_norm_consumer(g.ss, tid);
}

// SAFARA_TIMELINE builds: {start, end, smid | cycles << 16} of this CTA
// (thread 0 at the end of its role; consumers' warp 0 for compute CTAs).
__device__ __forceinline__ void ws_timeline(const Params &P, unsigned long long t_start,
                                            long long c_start) {
#ifdef SAFARA_TIMELINE
    if (P.dbg) {
        unsigned long long t_end;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
        unsigned smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        P.dbg[3 * blockIdx.x] = t_start;
        P.dbg[3 * blockIdx.x + 1] = t_end;
        P.dbg[3 * blockIdx.x + 2] = smid | ((unsigned long long)(clock64() - c_start) << 16);
    }
#else
    (void)P; (void)t_start; (void)c_start;
#endif
}

template <bool UD, bool AUX, bool NORM, bool PEER>
__device__ __forceinline__ void rhs_body_ws(const CUtensorMap *umap, const CUtensorMap *fmap,
                                            const Params &P) {
    unsigned long long t_start = 0;
    long long c_start = 0;
#ifdef SAFARA_TIMELINE
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_start));
    c_start = clock64();
#endif
    // PDL (SAFARA_PDL builds): the next pass on the stream may be scheduled
    // now; every global access below waits for the previous grid.
    grid_dep_launch();
    if (P.epoch) {  // f2: every CTA publishes "my u of this epoch is final"
        grid_dep_wait();
        peer_epoch_init(P);
        __syncthreads();
        peer_publish(P);
    }
    if ((int)blockIdx.x >= P.ncta) {  // the boundary faces (extra CTAs on idle SMs)
        grid_dep_wait();
        copy_faces<AUX>(P, (int)blockIdx.x - P.ncta, P.nface_cta);
        __syncthreads();
        if (threadIdx.x == 0) ws_timeline(P, t_start, c_start);
        peer_arrive(P);
        return;
    }
    const int tid = (int)threadIdx.x;
    if (tid == 0) {
        prefetch_tmap(umap);
        prefetch_tmap(fmap);
        for (int s = 0; s < WS_US; ++s) {
            mbar_init(&ws_full()[s], 1);
            mbar_init(&ws_afull()[s], WS_AW);
            mbar_init(&ws_empty()[s], TY);
        }
        for (int s = 0; s < WS_FS; ++s) {
            mbar_init(&ws_ffull()[s], 1);
            mbar_init(&ws_fempty()[s], TY);
        }
        fence_mbar_init();
    }
    __syncthreads();
    grid_dep_wait();
    if (P.nface_cta == 0) copy_faces<AUX>(P, (int)blockIdx.x, P.ncta);
    if (tid >= TY * 32) {
        setmaxnreg_dec_producer();
        ws_producer(umap, fmap, P);
        if (NORM) ws_norm_producer(P);
    } else {
        setmaxnreg_inc_consumer();
        ws_consumer<UD, AUX, NORM, PEER>(P);
        if (tid == 0) ws_timeline(P, t_start, c_start);
    }
    // f2: the grid completes only when no neighbour still reads our u (both
    // roles meet here; the peer loads were the consumers')
    peer_arrive(P);
}

}  // namespace dev
}  // namespace safara
