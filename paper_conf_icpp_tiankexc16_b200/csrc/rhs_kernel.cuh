// rhs_kernel.cuh -- the NAS BT/SP compute_rhs pass for sm_100a.
//
// Included by rhs_fast.cu (FMA contraction allowed, --fmad=true) and by
// rhs_strict.cu (--fmad=false: every product and sum rounded exactly where
// the NAS text rounds it, so the result is bit-identical to the oracle).
//
// Design:
//  * One thread per (i,j) column of a TX x TY CTA tile; the thread marches
//    along the sequential k loop.  This is SAFARA's split (PAPER.md
//    L684-692): the parallel i/j loops get no inter-iteration reuse, the
//    sequential k loop gets scalar replacement.
//  * Inter-iteration scalar replacement along k, prioritised by reuse
//    (cost model L x C): each u(m,i,j,k) is used at five
//    consecutive k steps.  The thread keeps u(:,i,j,k-1..k+1) plus its own
//    rho_i / square of the same planes in a register window (Fig. 6,
//    L895-914), and carries the zeta dissipation of plane k as the partial
//    ((u[k-2] - 4u[k-1]) + 6u[k]), formed one step early in the NAS order, in
//    place of a fifth plane.  The window rotates with period 3, so three
//    unrolled steps rotate it by register renaming alone (no moves; the
//    3-step body still fits the 32 KB instruction cache).
//  * i/j neighbours (reused by 4 other threads each, the "uncoalesced"
//    references SAFARA favours, L643-675) come from shared memory: the u
//    plane tile with a halo of 2 and the forcing tile arrive by TMA
//    (cp.async.bulk.tensor, STAGES-deep mbarrier ring refilled by the last
//    warp to release a slot).  rho_i / square of i+-1 come from the
//    neighbour lanes (shuffles), of j+-1 are recomputed from the u values
//    loaded for the stencil (rows belong to other warps; no cross-warp
//    wait).  Every other derived quantity (us, vs, ws, qs, u5*rho_i,
//    products) is recomputed at use from {u, rho_i, square}: one DMUL costs
//    a quarter of a shared-memory double (64 FP64 lanes vs 16 doubles/clk/SM).
//  * `dim`: u/forcing/rhs share one int32 descriptor (sy, sm, sk) held in the
//    kernel parameters (constant bank); `small`: all offsets are 32-bit.
//  * Evaluation order follows the NAS text left to right inside every
//    stencil difference (reading c6).  Where NAS multiplies by 2.0
//    or 4.0 (exact scalings) the subtract is a single fma, which rounds
//    identically.
#pragma once
#include <cstdio>
#include <type_traits>

#include "safara_internal.h"

// Production variant: the zeta (register-only) flux terms are accumulated
// first, while the xi/eta shared-memory loads are in flight, and the zeta
// dissipation last; STRICT keeps the NAS accumulation order forcing, xi,
// eta, zeta (reading c6).  Both are one accumulation chain per
// component.
#if SAFARA_STRICT_BUILD
#define SAFARA_ZETA_FIRST 0
#else
#ifndef SAFARA_ZETA_FIRST
#define SAFARA_ZETA_FIRST 1
#endif
#endif
#ifndef SAFARA_TMA_SPLIT
#define SAFARA_TMA_SPLIT 0  // 1: one TMA box per component (5 per field per plane)
#endif
#ifndef SAFARA_PROBE
#define SAFARA_PROBE 0  // roofline probes: 1 memory only, 2 compute only (no TMA waits/refills, no stores), 3 no rhs stores
#endif
#ifndef SAFARA_F_HINT
#define SAFARA_F_HINT 0  // 1: forcing TMA loads with an L2 evict_first hint
#endif
#ifndef SAFARA_U_HINT
#define SAFARA_U_HINT 0  // 1: u TMA loads with an L2 evict_last hint
#endif
#ifndef SAFARA_KBM_SMEM
#define SAFARA_KBM_SMEM 1  // unchecked-march bound read from shared memory each iteration
#endif
#ifndef SAFARA_PCHK_SPLIT
#define SAFARA_PCHK_SPLIT 1  // main k loop without the f2 peer-plane check (0: one loop, checked)
#endif
#ifndef SAFARA_XREG
#define SAFARA_XREG 1  // edge-tile xi case bits in a register (0: the smem table; A/B +-0.5 %)
#endif
#ifndef SAFARA_PDL
#define SAFARA_PDL 0  // programmatic dependent launch (see launch_pdl; A/B on B200: no gain, profiles/ab_pdl_r01.txt)
#endif
#ifndef SAFARA_STORE
#define SAFARA_STORE 0  // rhs stores: 0 st.global.cs, 1 default caching, 2 none (probe)
#endif
// Production reciprocal: 0 = seed + 3 Newton steps (6 DFMA), 1 = seed + 2
// Newton steps (4 DFMA), 2 = seed + one cubic step (3 DFMA; <= 1 ulp,
// profiles/rcp_ulp_r01.txt).
#ifndef SAFARA_RCP
#define SAFARA_RCP 2
#endif


namespace safara {
namespace dev {

// ---- `dim` / `small` ablation (Table I/II replica) ----------
// SAFARA_INDEX 0: one shared int32 descriptor for u/forcing/rhs (dim+small,
// production); 1: a separate int32 descriptor per array (small only);
// 2: separate int64 descriptors and 64-bit offsets per array (base).  The
// host fills every copy with the same values, so results are identical.
#ifndef SAFARA_INDEX
#define SAFARA_INDEX 0
#endif
#if SAFARA_INDEX == 0
typedef int idx_t;
#define SY(a) P.sy
#define SM(a) P.sm
#define SK(a) P.sk
#elif SAFARA_INDEX == 1
typedef int idx_t;
#define SY(a) P.a##_sy
#define SM(a) P.a##_sm
#define SK(a) P.a##_sk
#else
typedef long long idx_t;
#define SY(a) (long long)P.a##_sy64
#define SM(a) (long long)P.a##_sm64
#define SK(a) (long long)P.a##_sk64
#endif


constexpr int UPM = UX * UY;  // doubles per component plane of a u tile

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
                 : "memory");
}

__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    const uint32_t addr = smem_u32(bar);
    uint32_t done;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(addr), "r"(parity)
            : "memory");
    } while (!done);
}

// The same wait with a suspend-time hint: the waiting warp is parked (not
// spinning through try_wait / branch / yield) until the phase completes or
// `ns` elapses -- for warps whose wait is not on the critical path (the
// producer warpgroup of rhs_ws.cuh), so their spinning does not take issue
// slots from the consumers on the same SM sub-partition.
__device__ __forceinline__ void mbar_wait_sleep(uint64_t *bar, uint32_t parity, uint32_t ns) {
    const uint32_t addr = smem_u32(bar);
    uint32_t done;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(addr), "r"(parity), "r"(ns)
            : "memory");
    } while (!done);
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void tma_load_4d(void *dst, const CUtensorMap *map, uint64_t *bar,
                                            int c0, int c1, int c2, int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3),
        "r"(smem_u32(bar))
        : "memory");
}

// The same load with an L2 eviction-priority hint (createpolicy): forcing is
// read exactly once, so it can leave L2 first and leave room for the u halo
// rows that neighbouring tiles read again.
__device__ __forceinline__ void tma_load_4d_hint(void *dst, const CUtensorMap *map, uint64_t *bar,
                                                 int c0, int c1, int c2, int c3, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        ".L2::cache_hint [%0], [%1, {%2, %3, %4, %5}], [%6], %7;" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3),
        "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

__device__ __forceinline__ void tma_prefetch_l2_4d(const CUtensorMap *map, int c0, int c1, int c2,
                                                   int c3) {
    asm volatile(
        "cp.async.bulk.prefetch.tensor.4d.L2.global.tile [%0, {%1, %2, %3, %4}];" ::"l"(
            reinterpret_cast<uint64_t>(map)),
        "r"(c0), "r"(c1), "r"(c2), "r"(c3)
        : "memory");
}

// PDL: let the next grid on the stream be scheduled (its CTAs take SMs as
// ours exit and park in grid_dep_wait), and wait for the previous grid's
// completion before this grid's first global access.
__device__ __forceinline__ void grid_dep_launch() {
#if SAFARA_PDL
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
}
__device__ __forceinline__ void grid_dep_wait() {
#if SAFARA_PDL
    asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
}

__device__ __forceinline__ int reread(const int &x) {
    int r;
    asm volatile("mov.b32 %0, %1;" : "=r"(r) : "r"(x));
    return r;
}

__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

// ---- fused peer halo (include/safara.h safara_rhs_peer) ----
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long global_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// The pass's epoch: P.epoch, or with SAFARA_PEER_EPOCH_AUTO this rank's
// device counter + 1 (read by every CTA at its start, advanced by the last
// CTA at its end), so a CUDA graph of passes replays with fresh epochs.
__shared__ unsigned long long s_epoch;
__device__ __forceinline__ unsigned long long peer_epoch() { return s_epoch; }
__device__ __forceinline__ void peer_epoch_init(const Params &P) {
    if (threadIdx.x == 0)
        s_epoch = P.epoch == SAFARA_PEER_EPOCH_AUTO
                      ? *(volatile unsigned long long *)(P.pflags + SAFARA_PEER_EPOCH_WORD) + 1
                      : P.epoch;
}

// Acquire flag word `word` of this rank >= epoch.  Bounded wait: after
// P.peer_timeout_ns (SAFARA_PEER_TIMEOUT_MS, default 30 s) the wait is
// recorded in the flag words and the kernel TRAPS -- the caller's next
// synchronisation fails (cudaErrorLaunchFailure) instead of returning an rhs
// computed from a neighbour's stale planes, and a broken peer never hangs the
// GPU.
__device__ __forceinline__ void peer_wait(const Params &P, int word) {
    const unsigned long long e = peer_epoch();
    const unsigned long long *f = P.pflags + word;
    if (ld_acquire_sys(f) >= e) return;
    const unsigned long long t0 = global_ns();
    while (ld_acquire_sys(f) < e) {
        __nanosleep(200);
        if (global_ns() - t0 > P.peer_timeout_ns) {
            atomicAdd(P.pflags + SAFARA_PEER_TIMEOUTS, 1ull);
            atomicOr(P.pflags + SAFARA_PEER_TIMEOUT_WORDS, 1ull << word);  // which wait
            __threadfence_system();
            __trap();
        }
    }
}
// Own column (element offset colo = i + sy*j) of global plane kk, which lies
// outside the local range [pk_lo, pk_hi): a neighbour's owned plane, read over
// NVLink after acquiring its READY word.  These are the only values a slab
// needs from its neighbours (the zeta window); 0 beyond the global grid.
__device__ __forceinline__ void peer_col(double (&a)[5], const Params &P, int kk, int colo) {
    const bool lo = kk < P.pk_lo;
    const double *base = lo ? P.u_lo : P.u_hi;
    if (base == nullptr || kk < 0 || kk >= P.nz) {
#pragma unroll
        for (int m = 0; m < 5; ++m) a[m] = 0.0;
        return;
    }
    if (P.epoch) peer_wait(P, lo ? SAFARA_PEER_LO_READY : SAFARA_PEER_HI_READY);
    const double *p = base + (colo + SK(u) * (kk + (lo ? P.lo_koff : P.hi_koff)));
#pragma unroll
    for (int m = 0; m < 5; ++m) a[m] = __ldcg(p + SM(u) * m);
}
// Every CTA: this rank's u of this epoch is final (stream order) -- tell the
// neighbours.
__device__ __forceinline__ void peer_publish(const Params &P) {
    if (P.epoch == 0 || threadIdx.x != 0) return;
    const unsigned long long e = peer_epoch();
    __threadfence_system();
    if (P.pflags_lo) st_release_sys(P.pflags_lo + SAFARA_PEER_HI_READY, e);
    if (P.pflags_hi) st_release_sys(P.pflags_hi + SAFARA_PEER_LO_READY, e);
}
// Every CTA at exit (its peer loads are complete): the last one tells the
// neighbours we are done reading their u and waits until they are done with
// ours, so the grid completes only when u may be overwritten.
__device__ __forceinline__ void peer_arrive(const Params &P) {
    if (P.epoch == 0) return;
    __syncthreads();
    if (threadIdx.x != 0) return;
    const unsigned long long e = peer_epoch();
    __threadfence_system();
    const unsigned long long old = atomicAdd(P.pflags + SAFARA_PEER_ARRIVED, 1ull);
    if (old != (unsigned long long)gridDim.x - 1) return;
    P.pflags[SAFARA_PEER_ARRIVED] = 0;  // next epoch's grid is stream-ordered after us
    if (P.epoch == SAFARA_PEER_EPOCH_AUTO) P.pflags[SAFARA_PEER_EPOCH_WORD] = e;
    if (P.pflags_lo) st_release_sys(P.pflags_lo + SAFARA_PEER_HI_DONE, e);
    if (P.pflags_hi) st_release_sys(P.pflags_hi + SAFARA_PEER_LO_DONE, e);
    if (P.pflags_lo) peer_wait(P, SAFARA_PEER_LO_DONE);
    if (P.pflags_hi) peer_wait(P, SAFARA_PEER_HI_DONE);
}

// NAS second difference  (a[p] - 2.0*a[c]) + a[q]; 2.0*a[c] is exact, so the
// fused form rounds exactly like the two-step form.
__device__ __forceinline__ double d2(double ap, double ac, double aq) {
    return __fma_rn(-2.0, ac, ap) + aq;
}

// Reciprocal.  STRICT: IEEE 1.0/x (correctly rounded, bit-identical to the
// oracle).  Production: branch-free MUFU.RCP64H seed (about 20 good bits)
// refined by FMA steps (the IEEE division's special-case branch costs ~6
// issue slots per call; the densities of the path are normal and positive).
// The cubic step r*(1 + e + e^2), e = 1 - x*r, takes the seed error to ~2^-60
// before the final rounding (<= 1 ulp), in 3 DFMA instead of 2 Newton steps' 4.
__device__ __forceinline__ double recip(double x) {
#if SAFARA_STRICT_BUILD
    return 1.0 / x;
#else
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
#if SAFARA_RCP == 2
    const double e = __fma_rn(-x, r, 1.0);
    return __fma_rn(r, __fma_rn(e, e, e), r);
#else
    double e = __fma_rn(-x, r, 1.0);
    r = __fma_rn(r, e, r);
    e = __fma_rn(-x, r, 1.0);
#if SAFARA_RCP == 0
    r = __fma_rn(r, e, r);
    e = __fma_rn(-x, r, 1.0);
#endif
    return __fma_rn(r, e, r);
#endif
#endif
}

// rho_i = 1.0/u1; square = 0.5*(u2*u2 + u3*u3 + u4*u4)*rho_i  (App. A step 0)
__device__ __forceinline__ void aux_of(double u1, double u2, double u3, double u4, double &rho,
                                       double &sq) {
    rho = recip(u1);
    sq = 0.5 * (u2 * u2 + u3 * u3 + u4 * u4) * rho;
}

// the step-0 fields NAS x/y/z_solve consume, stored for
// the point at element offset `off` (i + sy*j) of local plane kl:
// rho_i, us, vs, ws, square, qs [, speed = sqrt(c1c2*rho_i*(u5 - square))].
__device__ __forceinline__ void store_aux(const Params &P, int off, int kl, double rho,
                                          double us, double vs, double ws, double sq,
                                          double qs, double u5) {
    double *a = P.aux + (off + P.ska * kl);
    const int sm = P.sm;
    __stcs(a, rho);
    __stcs(a + sm, us);
    __stcs(a + 2 * sm, vs);
    __stcs(a + 3 * sm, ws);
    __stcs(a + 4 * sm, sq);
    __stcs(a + 5 * sm, qs);
    if (P.naux > 6) __stcs(a + 6 * sm, sqrt(P.c.c1c2 * rho * (u5 - sq)));
}

struct Nb {
    double u[5];
    double rho, sq;
};

__device__ __forceinline__ Nb load_nb(const double *su, const double2 *sa, int uidx, int aidx) {
    Nb n;
#pragma unroll
    for (int m = 0; m < 5; ++m) n.u[m] = su[m * UPM + uidx];
    const double2 a = sa[aidx];
    n.rho = a.x;
    n.sq = a.y;
    return n;
}

__device__ __forceinline__ void load5(double (&a)[5], const double *su, int uidx) {
#pragma unroll
    for (int m = 0; m < 5; ++m) a[m] = su[m * UPM + uidx];
}

// Flux differences along one axis (App. A steps 2 / 4 / 6).  MOM = index of
// the momentum component along the axis (1 = xi, 2 = eta, 3 = zeta).
// `acc[m] = acc[m] + x`, or `acc[m] = x` for the first term of an independent
// partial sum (INIT): the production variant accumulates the directions in
// separate partial sums (shorter dependency chains; every stencil difference
// is still formed exactly in NAS order, reading c6).
template <bool INIT>
__device__ __forceinline__ double acc_add(double a, double x) {
    if (INIT) return x;
    return a + x;
}

template <int MOM, bool INIT, bool UD>
__device__ __forceinline__ void flux_dir(double (&acc)[5], const double (&cu)[5],
                                         const double (&vc)[3], double qsc, double pc,
                                         const Nb &p, const Nb &q, const Coef &C, int ax) {
    double vp[3], vq[3];
#pragma unroll
    for (int n = 0; n < 3; ++n) {
        vp[n] = p.u[n + 1] * p.rho;
        vq[n] = q.u[n + 1] * q.rho;
    }
    const double wp = vp[MOM - 1], wq = vq[MOM - 1], wc = vc[MOM - 1];
    const double t2 = C.t2[ax];

    acc[0] = acc_add<INIT>(acc[0], C.d1[ax][0] * d2(p.u[0], cu[0], q.u[0]));
    acc[0] = acc[0] - t2 * (p.u[MOM] - q.u[MOM]);
#pragma unroll
    for (int m = 1; m <= 3; ++m) {
        acc[m] = acc_add<INIT>(acc[m], C.d1[ax][UD ? 0 : m] * d2(p.u[m], cu[m], q.u[m]));
        if (m == MOM) {
            acc[m] = acc[m] + C.con2x43[ax] * d2(wp, wc, wq);
            acc[m] = acc[m] - t2 * ((p.u[m] * wp - q.u[m] * wq) +
                                    (((p.u[4] - p.sq) - q.u[4]) + q.sq) * C.c2);
        } else {
            acc[m] = acc[m] + C.con2[ax] * d2(vp[m - 1], vc[m - 1], vq[m - 1]);
            acc[m] = acc[m] - t2 * (p.u[m] * wp - q.u[m] * wq);
        }
    }
    acc[4] = acc_add<INIT>(acc[4], C.d1[ax][UD ? 0 : 4] * d2(p.u[4], cu[4], q.u[4]));
    acc[4] = acc[4] + C.con3[ax] * d2(p.sq * p.rho, qsc, q.sq * q.rho);
    acc[4] = acc[4] + C.con4[ax] * d2(wp * wp, wc * wc, wq * wq);
    acc[4] = acc[4] + C.con5[ax] * d2(p.u[4] * p.rho, pc, q.u[4] * q.rho);
    acc[4] = acc[4] - t2 * ((C.c1 * p.u[4] - C.c2 * p.sq) * wp -
                            (C.c1 * q.u[4] - C.c2 * q.sq) * wq);
}

// Fourth-order dissipation along one axis (App. A steps 3 / 5 / 7).  The
// GENERIC form covers all five NAS cases by zero-selecting the absent
// neighbours (exact: 0 - 4a = -4a, x + 0 = x) and choosing 5.0 or 6.0 for
// the centre; the non-generic form is the interior case only.
struct Cases {
    bool hm2, hm1, hp1, hp2, five;
};

__device__ __forceinline__ Cases cases_of(int x, int n) {
    Cases c;
    c.hm2 = x >= 3;
    c.hm1 = x >= 2;
    c.hp1 = x <= n - 3;
    c.hp2 = x <= n - 4;
    c.five = (x == 1) || (x == n - 2);
    return c;
}

// 3 <= x <= n-4 as one unsigned compare (n >= 6 is validated; n = 6 has no
// mid points)
__device__ __forceinline__ bool is_mid(int x, int n) {
    return (unsigned)(x - 3) < (unsigned)(n - 6);
}

// The dissipation stencil value t_m (before `rhs -= dssp*t`).  It is formed
// ahead of the flux terms (so the i+-2 / j+-2 neighbours die early: register
// pressure) and subtracted after them, keeping the NAS accumulation order.
template <bool GENERIC>
__device__ __forceinline__ void diss_terms(double (&t)[5], const double (&am2)[5],
                                           const double (&am1)[5], const double (&a0)[5],
                                           const double (&ap1)[5], const double (&ap2)[5],
                                           Cases cs) {
#pragma unroll
    for (int m = 0; m < 5; ++m) {
        if (!GENERIC) {
            t[m] = __fma_rn(-4.0, am1[m], am2[m]);
            t[m] = t[m] + 6.0 * a0[m];
            t[m] = __fma_rn(-4.0, ap1[m], t[m]);
            t[m] = t[m] + ap2[m];
        } else {
            const double x2 = cs.hm2 ? am2[m] : 0.0;
            const double x1 = cs.hm1 ? am1[m] : 0.0;
            const double y1 = cs.hp1 ? ap1[m] : 0.0;
            const double y2 = cs.hp2 ? ap2[m] : 0.0;
            const double cc = cs.five ? 5.0 * a0[m] : 6.0 * a0[m];
            t[m] = __fma_rn(-4.0, x1, x2);
            t[m] = t[m] + cc;
            t[m] = __fma_rn(-4.0, y1, t[m]);
            t[m] = t[m] + y2;
        }
    }
}

// The five NAS cases along i as ONE instruction sequence: the coefficients of
// a[i-1], a[i], a[i+1] come per lane from smem (-4/0, 6/5, -4/0) and an absent
// a[i-2] / a[i+2] is read from a zero-filled (out-of-box) column.  fma(0,x,y)
// = y, fma(-4,x,0) = -4x and c*a0 with c = 5 or 6 round exactly like the NAS
// expressions, so the result is bit-identical to the generic select form.
__device__ __forceinline__ void diss_terms_table(double (&t)[5], const double (&am2)[5],
                                                 const double (&am1)[5], const double (&a0)[5],
                                                 const double (&ap1)[5], const double (&ap2)[5],
                                                 double cm1, double c0, double cp1) {
#pragma unroll
    for (int m = 0; m < 5; ++m) {
        t[m] = __fma_rn(cm1, am1[m], am2[m]);
        t[m] = t[m] + c0 * a0[m];
        t[m] = __fma_rn(cp1, ap1[m], t[m]);
        t[m] = t[m] + ap2[m];
    }
}

// The five NAS cases along an axis whose case is warp-uniform (eta: one row
// per warp), each written out as the NAS text evaluates it -- uniform
// branches instead of per-element selects.  Case 0 is the interior form.
__device__ __forceinline__ void diss_terms_case(double (&t)[5], const double (&am2)[5],
                                                const double (&am1)[5], const double (&a0)[5],
                                                const double (&ap1)[5], const double (&ap2)[5],
                                                int c) {
    if (c == 0) {
#pragma unroll
        for (int m = 0; m < 5; ++m)
            t[m] = __fma_rn(-4.0, ap1[m], __fma_rn(-4.0, am1[m], am2[m]) + 6.0 * a0[m]) + ap2[m];
    } else if (c == 1) {  // 5a[x] - 4a[x+1] + a[x+2]
#pragma unroll
        for (int m = 0; m < 5; ++m) t[m] = __fma_rn(-4.0, ap1[m], 5.0 * a0[m]) + ap2[m];
    } else if (c == 2) {  // -4a[x-1] + 6a[x] - 4a[x+1] + a[x+2]
#pragma unroll
        for (int m = 0; m < 5; ++m)
            t[m] = __fma_rn(-4.0, ap1[m], -4.0 * am1[m] + 6.0 * a0[m]) + ap2[m];
    } else if (c == 3) {  // a[x-2] - 4a[x-1] + 6a[x] - 4a[x+1]
#pragma unroll
        for (int m = 0; m < 5; ++m)
            t[m] = __fma_rn(-4.0, ap1[m], __fma_rn(-4.0, am1[m], am2[m]) + 6.0 * a0[m]);
    } else {  // a[x-2] - 4a[x-1] + 5a[x]
#pragma unroll
        for (int m = 0; m < 5; ++m) t[m] = __fma_rn(-4.0, am1[m], am2[m]) + 5.0 * a0[m];
    }
}

__device__ __forceinline__ void diss_apply(double (&acc)[5], const double (&t)[5], double dssp) {
#pragma unroll
    for (int m = 0; m < 5; ++m) acc[m] = acc[m] - dssp * t[m];
}

// Face copy cache policy (experiments: SAFARA_FACE_CACHE 0 streaming .cs
// loads/stores, 1 .cg loads (L2 only) + .cs stores, 2 .cg loads + .cg stores)
#ifndef SAFARA_FACE_CACHE
#define SAFARA_FACE_CACHE 2
#endif
#if SAFARA_FACE_CACHE == 0
#define FACE_LD __ldcs
#define FACE_ST __stcs
#elif SAFARA_FACE_CACHE == 1
#define FACE_LD __ldcg
#define FACE_ST __stcs
#else
#define FACE_LD __ldcg
#define FACE_ST __stcg
#endif

// Copy forcing -> rhs on this launch's boundary-face points (rhs = forcing,
// unscaled; App. A step 1, reading c3), spread over all CTAs.
template <bool AUX>
__device__ __forceinline__ void copy_faces(const Params &P, int cta, int nctas) {
    const int nx = P.nx, ny = P.ny;
#ifdef SAFARA_PROBE_NO_IFACE
    const int per = 2 * nx;  // timing probe only: i-faces skipped
#else
    const int per = 2 * nx + 2 * (ny - 2);
#endif
    const int nloc = P.fk_hi - P.fk_lo;
    if (nloc <= 0) return;
    const long long nper = (long long)per * nloc;
    // full planes: global k == 0 or nz-1 inside [fk_lo, fk_hi)
    const int kl0 = 0 - P.k0, kl1 = (P.nz - 1) - P.k0;
    const bool has0 = kl0 >= P.fk_lo && kl0 < P.fk_hi;
    const bool has1 = kl1 >= P.fk_lo && kl1 < P.fk_hi;
    const int nfull = (int)has0 + (int)has1;
    const int full0 = has0 ? kl0 : kl1;  // first full plane; the second is always kl1
    const long long inner = (long long)(nx - 2) * (ny - 2);
    const long long total = nper + inner * nfull;
    // Batches of FB points per thread: all 5*FB loads are in flight before
    // the first store (one memory latency per batch, not per element).
    constexpr int FB = 4;
    const long long stride = (long long)nctas * blockDim.x;
    for (long long t0 = (long long)cta * blockDim.x + threadIdx.x; t0 < total;
         t0 += stride * FB) {
        int off[FB];
        double v[FB][5];
#pragma unroll
        for (int b = 0; b < FB; ++b) {
            const long long t = t0 + (long long)b * stride;
            off[b] = -1;
            if (t < total) {
                int i, j, kl;
                const int ti = (int)t;  // faces < 2^31 points (validated extents)
                if (t < nper) {
                    kl = P.fk_lo + ti / per;
                    int e = ti % per;
                    if (e < nx) {
                        i = e; j = 0;
                    } else if (e < 2 * nx) {
                        i = e - nx; j = ny - 1;
                    } else {
                        e -= 2 * nx;
                        if (e < ny - 2) { i = 0; j = 1 + e; }
                        else { i = nx - 1; j = 1 + e - (ny - 2); }
                        // written by the edge column tiles of this launch
                        if (P.iface_tiles && kl + P.k0 >= P.ka0 && kl + P.k0 < P.kb0) continue;
                    }
                } else {
                    const int e = ti - (int)nper;
                    kl = (e < inner) ? full0 : kl1;
                    const int r = e % (int)inner;
                    i = 1 + r % (nx - 2);
                    j = 1 + r / (nx - 2);
                }
                off[b] = i + SY(f) * j + SK(f) * kl;
#pragma unroll
                for (int m = 0; m < 5; ++m) v[b][m] = FACE_LD(P.f + off[b] + SM(f) * m);
                if (AUX) {  // aux of the face point from u (u plane = kl + ukoff)
                    const double *up = P.u + (i + SY(u) * j + SK(u) * (kl + P.ukoff));
                    const double u1 = __ldg(up), u2 = __ldg(up + SM(u)), u3 = __ldg(up + 2 * SM(u));
                    const double u4 = __ldg(up + 3 * SM(u)), u5 = __ldg(up + 4 * SM(u));
                    double rho, sq;
                    aux_of(u1, u2, u3, u4, rho, sq);
                    store_aux(P, i + P.sy * j, kl, rho, u2 * rho, u3 * rho, u4 * rho, sq,
                              sq * rho, u5);
                }
            }
        }
#pragma unroll
        for (int b = 0; b < FB; ++b)
            if (off[b] >= 0) {
#pragma unroll
                for (int m = 0; m < 5; ++m) FACE_ST(P.r + off[b] + SM(r) * m, v[b][m]);
            }
    }
}

__device__ __forceinline__ void issue_plane(const CUtensorMap *umap, const CUtensorMap *fmap,
                                            const Params &P, double *su, uint64_t *full, int i0,
                                            int j0, int k, bool with_f, uint32_t seq) {
    const int slot = (int)(seq % STAGES);
    if (k >= P.pk_hi) {  // f2: a neighbour's plane (own column read by peer_col)
        mbar_arrive(&full[slot]);
        return;
    }
    const int kb = k - P.k0 + P.ukoff;
    const int kf = k - P.k0;
    const int jc = j0 - 2;
    const int c1 = P.pos_j == 1 ? jc : (P.pos_m == 1 ? 0 : kb);
    const int c2 = P.pos_j == 2 ? jc : (P.pos_m == 2 ? 0 : kb);
    const int c3 = P.pos_j == 3 ? jc : (P.pos_m == 3 ? 0 : kb);
    double *dst = su + (size_t)slot * SLOT;
    mbar_expect_tx(&full[slot], with_f ? TMA_BYTES + TMA_BYTES_F : TMA_BYTES);
#if SAFARA_TMA_SPLIT
    // one box per component: more independent requests in flight per plane
    for (int m = 0; m < 5; ++m) {
        tma_load_4d(dst + m * UX * UY, umap, &full[slot], i0 - HX, P.pos_m == 1 ? m : c1,
                    P.pos_m == 2 ? m : c2, P.pos_m == 3 ? m : c3);
    }
#else
#if SAFARA_U_HINT == 1
    tma_load_4d_hint(dst, umap, &full[slot], i0 - HX, c1, c2, c3, policy_evict_last());
#else
    tma_load_4d(dst, umap, &full[slot], i0 - HX, c1, c2, c3);
#endif
#endif
    if (with_f) {
        const int f1 = P.pos_j == 1 ? j0 : (P.pos_m == 1 ? 0 : kf);
        const int f2 = P.pos_j == 2 ? j0 : (P.pos_m == 2 ? 0 : kf);
        const int f3 = P.pos_j == 3 ? j0 : (P.pos_m == 3 ? 0 : kf);
#if SAFARA_TMA_SPLIT
        for (int m = 0; m < 5; ++m)
            tma_load_4d(dst + U_SLOT + m * FX * TY, fmap, &full[slot], i0 - 1,
                        P.pos_m == 1 ? m : f1, P.pos_m == 2 ? m : f2, P.pos_m == 3 ? m : f3);
#else
#if SAFARA_F_HINT == 1
        tma_load_4d_hint(dst + U_SLOT, fmap, &full[slot], i0 - 1, f1, f2, f3, policy_evict_first());
#else
        tma_load_4d(dst + U_SLOT, fmap, &full[slot], i0 - 1, f1, f2, f3);
#endif
#endif
    }
}

// Warm L2 with plane k's u and forcing boxes (no smem, no barrier).
__device__ __forceinline__ void prefetch_plane_l2(const CUtensorMap *umap, const CUtensorMap *fmap,
                                                  const Params &P, int i0, int j0, int k,
                                                  bool with_f) {
    const int kb = k - P.k0 + P.ukoff;
    const int kf = k - P.k0;
    const int jc = j0 - 2;
    tma_prefetch_l2_4d(umap, i0 - HX, P.pos_j == 1 ? jc : (P.pos_m == 1 ? 0 : kb),
                       P.pos_j == 2 ? jc : (P.pos_m == 2 ? 0 : kb),
                       P.pos_j == 3 ? jc : (P.pos_m == 3 ? 0 : kb));
    if (with_f)
        tma_prefetch_l2_4d(fmap, i0 - 1, P.pos_j == 1 ? j0 : (P.pos_m == 1 ? 0 : kf),
                           P.pos_j == 2 ? j0 : (P.pos_m == 2 ? 0 : kf),
                           P.pos_j == 3 ? j0 : (P.pos_m == 3 ? 0 : kf));
}

__device__ __forceinline__ void wait_plane(uint64_t *full, uint32_t seq) {
    mbar_wait(&full[seq % STAGES], (seq / STAGES) & 1u);
}

// Decode linear column-plane unit L (chunk-major: all column tiles advance
// through the same band of k-planes together, so a plane's i/j halo that a
// neighbouring tile fetched is still in L2) into (column, plane index) and the
// number of units left in this (chunk, column) run.
// floor(c * units / ncta) without a 64-bit division subroutine call (keeps
// the loop control visibly warp-uniform, so shuffles need no collective path)
__device__ __forceinline__ int split_point(int c, int units, int ncta) {
    const long long num = (long long)c * units;
    long long q = (long long)((double)num / (double)ncta);
    while (q * ncta > num) --q;
    while ((q + 1) * ncta <= num) ++q;
    return (int)q;
}

__device__ __forceinline__ void decode_unit(const Params &P, int L, int &col, int &pidx,
                                            int &run) {
    const int per_chunk = P.chunk * P.ncol;
    const int c = L / per_chunk;
    const int rem = L - c * per_chunk;
    const int kc = min(P.chunk, P.nplanes - c * P.chunk);
    col = rem / kc;
    const int off = rem - col * kc;
    pidx = c * P.chunk + off;
    run = kc - off;
}

// The segment starting at unit ub (not crossing a column, a plane range or
// the CTA's end ue): column tile `col`, global planes [ka, kb).
__device__ __forceinline__ void segment_of(const Params &P, int ub, int ue, int &col, int &ka,
                                           int &kb) {
    int pidx, run;
    decode_unit(P, ub, col, pidx, run);
    const int left = min(run, ue - ub);
    if (pidx < P.n0) {
        ka = P.ka0 + pidx;
        kb = min(P.kb0, ka + left);
    } else {
        ka = P.ka1 + (pidx - P.n0);
        kb = min(P.kb1, ka + left);
    }
}

// Per-segment state of one thread: the register window of the k march.
// At rotation R (= step index mod 3) plane k-1 lives in a[R], plane k in
// a[(R+1)%3] and plane k+1 in a[(R+2)%3]; plane k+2 is loaded into a[R] once
// plane k-1 is dead, so three unrolled steps rotate the window by register
// renaming alone (no moves).  The zeta dissipation of plane k is carried as
// its partial ((a[k-2] - 4a[k-1]) + 6a[k]) -- formed one step early, in the
// NAS order -- instead of keeping a fifth plane a[k-2].
// Shared-memory carve-up (addresses are link-time constants, so nothing here
// occupies a register across the loop).
extern __shared__ __align__(128) unsigned char smem_raw[];
__device__ __forceinline__ double *smem_ring() { return reinterpret_cast<double *>(smem_raw); }
__device__ __forceinline__ uint64_t *smem_full() {
    return reinterpret_cast<uint64_t *>(smem_ring() + (size_t)STAGES * SLOT);
}
__device__ __forceinline__ unsigned int *smem_released() {
    return reinterpret_cast<unsigned int *>(smem_full() + STAGES);
}
// Per-lane xi-dissipation coefficients of the current column tile:
// [0][lane] = coefficient of a[i-1] (-4 or 0), [1][lane] = of a[i] (6 or 5),
// [2][lane] = of a[i+1] (-4 or 0).
__device__ __forceinline__ double *smem_xcoef() {
    return reinterpret_cast<double *>(smem_ring() + (size_t)STAGES * SLOT + XCOEF_OFF);
}

// This CTA's unit range [ub, ue) and the current segment's end plane kb
// live in shared memory across the k march (CTA-uniform; keeps registers free
// for the unrolled window).
__shared__ int s_range[8];  // ub, ue, segment kb, next segment's ub, tile i0, j0, segment ka,
                            // end of the unchecked k march (min(kb, pk_hi - 2))
__device__ __forceinline__ int smem_kb() { return *(volatile int *)&s_range[2]; }

struct Seg {
    double *rptr;  // rhs of (i, j, k, m=0) for the current step
    int ka, kb;
    int uc;         // own column's element offset in the u tile
    int fo;         // own column's element offset in the forcing tile (= ty*FX + tx + 1)
    bool lane0, lane31;
    bool active, mid_x;
    int ycase;      // NAS dissipation case of row j: 0 mid, 1 j=1, 2 j=2, 3 j=ny-3, 4 j=ny-2
#if SAFARA_XREG
    int xo;         // edge tiles: i+-2 offsets and xi-dissipation case bits of this lane
#endif
    uint32_t seq0;  // ring sequence number of the segment's first plane
    double a[3][5];      // u(:, i, j, k-1..k+1), rotating (see above)
    double ra[3], sa[3]; // rho_i / square of the same planes
    double tp[5];        // zeta dissipation partial of plane k
};

// The zeta dissipation partial of plane kk: ((x2 - 4 x1) + c0 a0) with the
// NAS case of kk selecting which neighbours exist (exact zero selection).
__device__ __forceinline__ void zeta_partial(double (&tp)[5], const double (&am2)[5],
                                             const double (&am1)[5], const double (&a0)[5],
                                             int kk, int nz, bool mid) {
    if (mid) {
#pragma unroll
        for (int m = 0; m < 5; ++m) tp[m] = __fma_rn(-4.0, am1[m], am2[m]) + 6.0 * a0[m];
    } else {
        const Cases c = cases_of(kk, nz);
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            const double x2 = c.hm2 ? am2[m] : 0.0;
            const double x1 = c.hm1 ? am1[m] : 0.0;
            const double cc = c.five ? 5.0 * a0[m] : 6.0 * a0[m];
            tp[m] = __fma_rn(-4.0, x1, x2) + cc;
        }
    }
}

// PCHK: plane k+2 may lie beyond the local slab (f2 peer halo; only the
// last steps of a slab's march are instantiated with the check).
template <int R, bool UD, bool AUX, bool PCHK>
__device__ __forceinline__ void rhs_step(Seg &g, const Params &P, const CUtensorMap *umap,
                                         const CUtensorMap *fmap, int k) {
    constexpr int Q = R % 3, Z = (R + 1) % 3, PI = (R + 2) % 3;  // planes k-1, k, k+1
    const unsigned FULL = 0xffffffffu;
    if (PCHK && k >= g.kb) return;  // single-loop march: past the segment end
#ifdef SAFARA_STEPLOG
    if (threadIdx.x == 0 && P.steplog && k - g.ka < 126)
        P.steplog[blockIdx.x * 128 + 2 + (k - g.ka)] = global_ns();
#endif
    const Coef &C = P.c;
    const uint32_t sq_k = g.seq0 + (uint32_t)(k - g.ka);  // ring sequence number of plane k
    double *const su = smem_ring();
    const double *s = su + (size_t)(sq_k % STAGES) * SLOT;

    // forcing(k): staged by the same TMA as plane k (reuse count 1, so it only
    // needs latency hiding, not a register slot)
    unsigned rel_old = 0;  // slot-release counter value seen by lane 0
    double acc[5];
    {
        const double *fs = s + U_SLOT;
#pragma unroll
        for (int m = 0; m < 5; ++m) acc[m] = fs[m * TY * FX + g.fo];
    }
    // plane k+2 must have landed: its own column enters the window at the
    // end of this step (read from smem there, so it holds no registers
    // across the step); own rho_i / square of plane k+1
    if (SAFARA_PROBE != 2) wait_plane(smem_full(), sq_k + 2);
    const double *const s2 = su + (size_t)((sq_k + 2) % STAGES) * SLOT;
    aux_of(g.a[PI][0], g.a[PI][1], g.a[PI][2], g.a[PI][3], g.ra[PI], g.sa[PI]);

    double an[5];
#if SAFARA_PROBE == 1
    load5(an, s2, g.uc);
#pragma unroll
    for (int m = 0; m < 5; ++m) acc[m] = acc[m] + an[m] * g.ra[PI] + s[g.uc + m * UPM];
    __syncwarp();
    if (g.lane0) {
        __threadfence_block();
        rel_old = atomicAdd(&smem_released()[(int)(sq_k % STAGES)], 1u);
    }
#else
    const double (&wz)[5] = g.a[Z];
    const double r0 = g.ra[Z], s0 = g.sa[Z];
    double vc[3];
    vc[0] = wz[1] * r0;
    vc[1] = wz[2] * r0;
    vc[2] = wz[3] * r0;
    const double qsc = s0 * r0;
    const double pc = wz[4] * r0;
    if (AUX && g.active) {
        // element offset of (i, j) from the walking rhs pointer
        const int kl = k - P.k0;
        const int off = (int)(g.rptr - P.r) - SK(r) * kl;
        store_aux(P, off, kl, r0, vc[0], vc[1], vc[2], s0, qsc, wz[4]);
    }

    // zeta dissipation of plane k: the carried partial completed with
    // u(k+1) and u(k+2) (uniform branch: edge planes only)
    auto zeta_diss = [&](double (&t_z)[5]) {
        if (is_mid(k, P.nz)) {
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
    };
    auto zeta = [&]() {
        Nb p, q;
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            p.u[m] = g.a[PI][m];
            q.u[m] = g.a[Q][m];
        }
        p.rho = g.ra[PI]; p.sq = g.sa[PI];
        q.rho = g.ra[Q]; q.sq = g.sa[Q];
        flux_dir<3, false, UD>(acc, wz, vc, qsc, pc, p, q, C, 2);
    };
#if SAFARA_ZETA_FIRST
    // zeta: everything from the register window (inter-iteration scalar
    // replacement along the sequential loop), while the xi/eta shared-memory
    // loads are in flight
    zeta();
#endif
    // xi: rho_i/square of i+-1 are the neighbour lanes' own values; lanes 0
    // and 31 evaluate their outside neighbour themselves.
    {
        Nb p, q;
        load5(p.u, s, g.uc + 1);
        load5(q.u, s, g.uc - 1);
        p.rho = __shfl_down_sync(FULL, r0, 1);
        p.sq = __shfl_down_sync(FULL, s0, 1);
        q.rho = __shfl_up_sync(FULL, r0, 1);
        q.sq = __shfl_up_sync(FULL, s0, 1);
        {
            const bool left = g.lane0;
            double re, se;
            aux_of(left ? q.u[0] : p.u[0], left ? q.u[1] : p.u[1], left ? q.u[2] : p.u[2],
                   left ? q.u[3] : p.u[3], re, se);
            if (left) { q.rho = re; q.sq = se; }
            if (g.lane31) { p.rho = re; p.sq = se; }
        }
        double t[5];
        {
            double pp[5], qq[5];
            if (g.mid_x) {
                load5(pp, s, g.uc + 2);
                load5(qq, s, g.uc - 2);
                diss_terms<false>(t, qq, q.u, wz, p.u, pp, Cases{});
            } else {
                // edge tile: absent i-2 / i+2 -> the zero-filled column beyond
                unsigned lane;  // = tx
                asm("mov.u32 %0, %%laneid;" : "=r"(lane));
#if SAFARA_XREG
                // per-lane case bits held in one register (no table loads)
                const int xo = g.xo;
                load5(pp, s, g.uc + (xo & 0xff));
                load5(qq, s, g.uc - ((xo >> 8) & 0xff));
                diss_terms_table(t, qq, q.u, wz, p.u, pp, (xo & (1 << 16)) ? -4.0 : 0.0,
                                 (xo & (1 << 17)) ? 5.0 : 6.0, (xo & (1 << 18)) ? -4.0 : 0.0);
                (void)lane;
#else
                const double *xc = smem_xcoef();
                const int xo = reinterpret_cast<const int *>(xc + 3 * TX)[lane];
                load5(pp, s, g.uc + (xo & 0xff));
                load5(qq, s, g.uc - (xo >> 8));
                diss_terms_table(t, qq, q.u, wz, p.u, pp, xc[lane], xc[TX + lane],
                                 xc[2 * TX + lane]);
#endif
            }
        }
        flux_dir<1, false, UD>(acc, wz, vc, qsc, pc, p, q, C, 0);
        diss_apply(acc, t, C.dssp);
    }
    // eta: rows j+-1 belong to other warps; evaluate their rho_i / square
    // from the u values loaded for the stencil (no cross-warp dependency)
    {
        Nb p, q;
        load5(p.u, s, g.uc + UX);
        load5(q.u, s, g.uc - UX);
        aux_of(p.u[0], p.u[1], p.u[2], p.u[3], p.rho, p.sq);
        aux_of(q.u[0], q.u[1], q.u[2], q.u[3], q.rho, q.sq);
        double t[5];
        {
            double pp[5], qq[5];
            load5(pp, s, g.uc + 2 * UX);
            load5(qq, s, g.uc - 2 * UX);
            diss_terms_case(t, qq, q.u, wz, p.u, pp, g.ycase);
        }
        // Every read of plane k's slot is done: release it now, act on the
        // counter at the end of the step (its latency hides behind eta).
        __syncwarp();
        if (g.lane0) {
            __threadfence_block();
            rel_old = atomicAdd(&smem_released()[(int)(sq_k % STAGES)], 1u);
        }
        flux_dir<2, false, UD>(acc, wz, vc, qsc, pc, p, q, C, 1);
        diss_apply(acc, t, C.dssp);
    }
#if !SAFARA_ZETA_FIRST
    zeta();
#endif
    // u(k+2) completes the zeta dissipation of plane k (production applies
    // it last, STRICT right after the zeta fluxes -- the NAS order)
    if (!PCHK || k + 2 < P.pk_hi) {
        load5(an, s2, g.uc);
    } else {  // f2: plane k+2 belongs to the upper neighbour
        unsigned lane;
        asm("mov.u32 %0, %%laneid;" : "=r"(lane));
        const int i = min(s_range[4] + (int)lane, P.nx - 1);
        const int j = min(s_range[5] + (int)(threadIdx.x / TX), P.ny - 1);
        peer_col(an, P, k + 2, i + P.sy * j);
    }
    {
        double t_z[5];
        zeta_diss(t_z);
        diss_apply(acc, t_z, C.dssp);
    }
#endif  // SAFARA_PROBE == 1
    if (g.active && ((SAFARA_PROBE != 3 && SAFARA_PROBE != 2) || acc[0] == 1.2345e300)) {
        // rptr walks down the column one plane per step; the 5 component
        // planes are sm apart (one 64-bit pointer instead of 5 addresses)
        double *rp = g.rptr;
#pragma unroll
        for (int m = 0; m < 5; ++m) {
#if SAFARA_STORE == 0
            __stcs(rp, acc[m] * C.dt);
#elif SAFARA_STORE == 1
            *rp = acc[m] * C.dt;
#else
            if (acc[m] == 1.2345e300) *rp = acc[m];
#endif
            rp += SM(r);
        }
    }
    g.rptr += SK(r);
    // the zeta partial of plane k+1 (plane k-1's last use), then rotate by
    // renaming: plane k+2 takes the dead plane k-1's slot
#if SAFARA_PROBE != 1
    zeta_partial(g.tp, g.a[Q], g.a[Z], g.a[PI], k + 1, P.nz, is_mid(k + 1, P.nz));
#endif
#pragma unroll
    for (int m = 0; m < 5; ++m) g.a[Q][m] = an[m];
    // the last warp out of plane k (see the release above) refills its slot
    if (SAFARA_PROBE != 2 && g.lane0 && rel_old == (unsigned)(TY - 1)) {
        smem_released()[(int)(sq_k % STAGES)] = 0;
        __threadfence_block();
        const int kn = k + STAGES, kb = smem_kb();  // segment end (read rarely)
        if (kn <= kb + 1)
            issue_plane(umap, fmap, P, su, smem_full(), s_range[4], s_range[5], kn, kn < kb,
                        sq_k + STAGES);
    }
}

// One CTA processes the column-plane units [blockIdx*units/ncta, ...).
// Warps are decoupled: warp w owns row j0+w of the tile and never waits for
// another warp except through the TMA ring (a slot is refilled by the last
// warp to release it).
// UD: the host verified dX1..dX5 are equal per axis (true for NAS), so one
// d1 coefficient per axis suffices -- fewer uniform registers to reload.
// ONE: the single-loop march (slabs with an upper peer, see below).
template <bool UD, bool AUX, bool ONE>
__device__ __forceinline__ void rhs_body(const CUtensorMap *umap, const CUtensorMap *fmap,
                                         const Params &P) {
#ifdef SAFARA_TIMELINE
    unsigned long long t_start;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_start));
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    const long long c_start = clock64();
#endif
    // Extra CTAs beyond the compute grid (on SMs the lockstep schedule leaves
    // idle) only copy the boundary faces.
    grid_dep_launch();
    if (P.epoch) {
        // after the previous grid (PDL): its writes to u are complete before
        // READY is published, and its epoch advance is visible
        grid_dep_wait();
        peer_epoch_init(P);
        __syncthreads();
        peer_publish(P);
    }
    if ((int)blockIdx.x >= P.ncta) {
        grid_dep_wait();
        copy_faces<AUX>(P, (int)blockIdx.x - P.ncta, P.nface_cta);
        peer_arrive(P);
#ifdef SAFARA_TIMELINE
        if (threadIdx.x == 0 && P.dbg) {
            unsigned long long t_end;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
            P.dbg[3 * blockIdx.x] = t_start;
            P.dbg[3 * blockIdx.x + 1] = t_end;
            P.dbg[3 * blockIdx.x + 2] = smid | ((unsigned long long)(clock64() - c_start) << 16);
        }
#endif
        return;
    }
    double *su = smem_ring();
    uint64_t *full = smem_full();
    unsigned int *released = smem_released();

    const int tid = threadIdx.x;

    if (tid == 0) {
        prefetch_tmap(umap);
        prefetch_tmap(fmap);
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&full[s], 1);
            released[s] = 0;
        }
        fence_mbar_init();
    }
    __syncthreads();
    grid_dep_wait();

    int ub, ue;
    if (P.parts > 0) {
        // lockstep: CTA c owns column tile c % ncol, k-part c / ncol (all
        // parts of one plane band run on CTAs spread over the whole chip)
        const int c = (int)blockIdx.x, col = c % P.ncol, part = c / P.ncol;
        // split_bias: the last part is made shorter by that many planes (its
        // final steps wait for the upper peer's planes, f2), the others share them
        const int np = P.nplanes + P.split_bias;
        ub = col * P.nplanes + max(0, min((part * np) / P.parts, P.nplanes));
        ue = col * P.nplanes + (part + 1 == P.parts ? P.nplanes
                                                     : max(0, min(((part + 1) * np) / P.parts,
                                                                  P.nplanes)));
    } else {
        ub = split_point((int)blockIdx.x, P.units, P.ncta);
        ue = split_point((int)blockIdx.x + 1, P.units, P.ncta);
    }

    Seg g;
    g.lane0 = tid % TX == 0;
    g.lane31 = tid % TX == TX - 1;
    g.fo = (tid / TX) * FX + tid % TX + 1;
    g.seq0 = 0;

    // The first segment's planes are requested before the boundary-face copy
    // so that the copy overlaps their latency.
    bool first = true;
    if (ub < ue && tid == 0) {
        int col, ka, kb;
        segment_of(P, ub, ue, col, ka, kb);
        const int nload = kb - ka + 2;
        const int npre = nload < STAGES ? nload : STAGES;
        const int i0 = 1 + (col % P.ntx) * TX, j0 = 1 + (col / P.ntx) * TY;
        for (int s = 0; s < npre; ++s)
            issue_plane(umap, fmap, P, su, full, i0, j0, ka + s, ka + s < kb, (uint32_t)s);
    }
    if (P.nface_cta == 0) copy_faces<AUX>(P, (int)blockIdx.x, P.ncta);

    if (tid == 0) {
        s_range[0] = ub;
        s_range[1] = ue;
    }
    __syncthreads();
    while (true) {
        // ---- segment: one column tile, a contiguous run of planes ----
        ub = *(volatile int *)&s_range[0];
        ue = *(volatile int *)&s_range[1];
        if (ub >= ue) break;
        int col;
        segment_of(P, ub, ue, col, g.ka, g.kb);
        // (re-read rather than kept live across the march)
        unsigned tid_r;
        asm volatile("mov.u32 %0, %%tid.x;" : "=r"(tid_r));
        const int tx = (int)tid_r % TX, ty = (int)tid_r / TX;  // lane = tx, warp = ty
        const int i0 = 1 + (col % P.ntx) * TX, j0 = 1 + (col / P.ntx) * TY;
        if (tid == 0) {  // read by the refilling lane / at the segment end
            s_range[2] = g.kb;
            s_range[3] = ub + (g.kb - g.ka);
            s_range[4] = i0;
            s_range[5] = j0;
            s_range[6] = g.ka;
            s_range[7] = min(g.kb, P.pk_hi - 2);
        }
        const int ka = g.ka, kb = g.kb;

        const int i = i0 + tx, j = j0 + ty;
        // extents re-read per segment (volatile: not hoisted into registers
        // live across the march)
        const int nx_s = reread(P.nx), ny_s = reread(P.ny);
        g.active = (i <= nx_s - 2) && (j <= ny_s - 2);
        const int nload = kb - ka + 2;  // ring planes ka .. kb+1

        if (tid == 0 && !first) {
            const int npre = nload < STAGES ? nload : STAGES;
            for (int s = 0; s < npre; ++s)
                issue_plane(umap, fmap, P, su, full, i0, j0, ka + s, ka + s < kb, g.seq0 + s);
        }
        first = false;

        // Case flags (global indices, reading c12).
        g.mid_x = is_mid(i0, P.nx) && is_mid(i0 + TX - 1, P.nx);
        if (!g.mid_x && tid < TX) {
            const Cases cs = cases_of(i0 + tid, P.nx);
            double *xc = smem_xcoef();
            xc[tid] = cs.hm1 ? -4.0 : 0.0;
            xc[TX + tid] = cs.five ? 5.0 : 6.0;
            xc[2 * TX + tid] = cs.hp1 ? -4.0 : 0.0;
            // offsets of a[i+2] / a[i-2], redirected to the zero-filled column
            // beyond the box where NAS drops the term
            reinterpret_cast<int *>(xc + 3 * TX)[tid] =
                (i0 + tid == P.nx - 3 ? 3 : 2) | ((i0 + tid == 2 ? 3 : 2) << 8);
        }
        if (!g.mid_x) __syncthreads();  // the coefficient table is CTA-wide
#if SAFARA_XREG
        {
            const Cases cs = cases_of(i0 + tx, P.nx);
            g.xo = (i0 + tx == P.nx - 3 ? 3 : 2) | ((i0 + tx == 2 ? 3 : 2) << 8) |
                   (cs.hm1 ? 1 << 16 : 0) | (cs.five ? 1 << 17 : 0) | (cs.hp1 ? 1 << 18 : 0);
        }
#endif
        g.ycase = is_mid(j, ny_s) ? 0 : j == 1 ? 1 : j == 2 ? 2 : j == ny_s - 3 ? 3 : 4;
        g.uc = (ty + 2) * UX + (tx + HX);  // centre in the u tile
        g.rptr = P.r + ((idx_t)i + SY(r) * j + SK(r) * (ka - P.k0));

        // Window at rotation 0: planes ka-2 (only for the zeta partial) and
        // ka-1 from global memory (read once per segment), ka and ka+1 from
        // the TMA ring.  Lanes outside the grid read the nearest in-grid
        // column (valid memory; they store nothing and feed no active lane).
        {
            const int ic = min(i, nx_s - 1), jc = min(j, ny_s - 1);
            const int lk = ka - P.k0 + P.ukoff;  // local u plane of ka
            const double *uc0 = P.u + (idx_t)(ic + SY(u) * jc);
            const int colo = ic + P.sy * jc;
            if (ka - 1 < P.pk_lo) {
                peer_col(g.a[0], P, ka - 1, colo);
            } else {
#pragma unroll
                for (int m = 0; m < 5; ++m)
                    g.a[0][m] = lk - 1 >= 0 ? __ldg(uc0 + SM(u) * m + SK(u) * (lk - 1)) : 0.0;
            }
            wait_plane(full, g.seq0);
            load5(g.a[1], su + (size_t)(g.seq0 % STAGES) * SLOT, g.uc);
            {
                double am2[5];
                if (ka - 2 < P.pk_lo) {
                    peer_col(am2, P, ka - 2, colo);
                } else {
#pragma unroll
                    for (int m = 0; m < 5; ++m)
                        am2[m] = lk - 2 >= 0 ? __ldg(uc0 + SM(u) * m + SK(u) * (lk - 2)) : 0.0;
                }
                zeta_partial(g.tp, am2, g.a[0], g.a[1], ka, P.nz, is_mid(ka, P.nz));
            }
            aux_of(g.a[0][0], g.a[0][1], g.a[0][2], g.a[0][3], g.ra[0], g.sa[0]);
            aux_of(g.a[1][0], g.a[1][1], g.a[1][2], g.a[1][3], g.ra[1], g.sa[1]);
            wait_plane(full, g.seq0 + 1);
            if (ka + 1 < P.pk_hi)
                load5(g.a[2], su + (size_t)((g.seq0 + 1) % STAGES) * SLOT, g.uc);
            else
                peer_col(g.a[2], P, ka + 1, colo);
        }

        int k = ka;
        if (ONE) {
            // slabs with an upper peer (f2): one warm checked 3-step body for
            // the whole march, steps past kb return at once -- no separately
            // compiled tail code, which runs cold (fetched from HBM: the
            // streaming data has flushed L2) and cost C/8 slabs 2-3 us a pass
#pragma unroll 1
            for (; k < kb; k += 3) {
                rhs_step<0, UD, AUX, true>(g, P, umap, fmap, k);
                rhs_step<1, UD, AUX, true>(g, P, umap, fmap, k + 1);
                rhs_step<2, UD, AUX, true>(g, P, umap, fmap, k + 2);
            }
        } else {
        // steps whose plane k+2 is local (all of them unless the slab's upper
        // neighbour is a peer, f2) run without the peer check
#if SAFARA_PCHK_SPLIT
#pragma unroll 1
#if SAFARA_KBM_SMEM
        for (; k + 3 <= *(volatile int *)&s_range[7]; k += 3) {
#else
        for (; k + 3 <= min(smem_kb(), P.pk_hi - 2); k += 3) {
#endif
            rhs_step<0, UD, AUX, false>(g, P, umap, fmap, k);
            rhs_step<1, UD, AUX, false>(g, P, umap, fmap, k + 1);
            rhs_step<2, UD, AUX, false>(g, P, umap, fmap, k + 2);
        }
#endif
#pragma unroll 1
        for (; k + 3 <= smem_kb(); k += 3) {
            rhs_step<0, UD, AUX, true>(g, P, umap, fmap, k);
            rhs_step<1, UD, AUX, true>(g, P, umap, fmap, k + 1);
            rhs_step<2, UD, AUX, true>(g, P, umap, fmap, k + 2);
        }
        if (k < kb) {
            rhs_step<0, UD, AUX, true>(g, P, umap, fmap, k);
            if (k + 1 < kb) rhs_step<1, UD, AUX, true>(g, P, umap, fmap, k + 1);
        }
        }
        g.seq0 += (uint32_t)(s_range[2] - s_range[6] + 2);  // planes ka .. kb+1
        // Segment end: every warp has consumed every plane; planes kb, kb+1
        // were never released, so clear the counters before the next segment.
        __syncthreads();
        if (tid < STAGES) released[tid] = 0;
        if (tid == 0) s_range[0] = s_range[3];
        __syncthreads();
    }
    peer_arrive(P);
#ifdef SAFARA_TIMELINE
    if (tid == 0 && P.dbg) {
        unsigned long long t_end;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
        P.dbg[3 * blockIdx.x] = t_start;
        P.dbg[3 * blockIdx.x + 1] = t_end;
        P.dbg[3 * blockIdx.x + 2] = smid | ((unsigned long long)(clock64() - c_start) << 16);
    }
#endif
}

}  // namespace dev
}  // namespace safara
