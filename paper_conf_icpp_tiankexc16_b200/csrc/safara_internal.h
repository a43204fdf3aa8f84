// safara_internal.h -- types shared by the host ABI (api.cu) and the kernel
// translation units (rhs_fast.cu / rhs_strict.cu).  Not part of the C ABI.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "safara.h"

namespace safara {

// CTA tile: TX x TY (i, j) columns, one thread per column marching along k.
constexpr int TX = 32;
#ifndef SAFARA_TY
#define SAFARA_TY 12
#endif
constexpr int TY = SAFARA_TY;
constexpr int NTHREADS = TX * TY;
#ifndef SAFARA_STAGES
#define SAFARA_STAGES 4
#endif
constexpr int STAGES = SAFARA_STAGES;  // planes in the TMA ring
// u tile: i halo of 2 plus one pad column each side.  The TMA box's first
// element must be 16-byte aligned (fp64: even i), and tiles start at odd i
// (interior begins at i = 1), so the box starts at i0 - 3 and is TX + 6 wide.
constexpr int HX = 3;                // u-tile column of the tile's first i
constexpr int UX = TX + 2 * HX;
constexpr int UY = TY + 4;           // u tile incl. j halo of 2
constexpr int U_PLANE = UX * UY * 5; // doubles in one TMA box (one u plane tile)
constexpr int U_SLOT = ((U_PLANE * 8 + 127) / 128) * 128 / 8;  // slot stride: TMA dst 128 B aligned
constexpr uint32_t TMA_BYTES = U_PLANE * 8u;
// forcing tile of the same plane: i0-1 .. i0+TX (16-byte aligned start), no j halo
constexpr int FX = TX + 2;
constexpr int F_PLANE = FX * TY * 5;
constexpr int F_SLOT = ((F_PLANE * 8 + 127) / 128) * 128 / 8;
constexpr uint32_t TMA_BYTES_F = F_PLANE * 8u;
constexpr int SLOT = U_SLOT + F_SLOT;  // doubles per ring slot: u tile then forcing tile
constexpr int XCOEF_OFF = 16;  // doubles after the ring: mbarriers + counters first
static_assert(STAGES * (8 + 4) <= XCOEF_OFF * 8, "mbarriers + release counters fit before the table");
// after the mbarriers: the edge-tile xi table, 3 coefficient rows (double)
// and one row of packed i+-2 offsets (int)
constexpr size_t SMEM_BYTES = (size_t)STAGES * SLOT * 8 + (XCOEF_OFF + 3 * TX + TX / 2) * 8;
constexpr int MIN_PLANES_PER_CTA = 2;  // small slabs: more k-parts win (SP-B/8: 16.4 -> 12.5 us, profiles/slab_sim_r01.txt)

// Round 2 warp-specialised kernel (rhs_ws.cuh): TY consumer warps + one
// producer warpgroup; u / aux / forcing rings in shared memory.
constexpr int WS_PW = 4;                     // producer warps (one warpgroup)
constexpr int WS_THREADS = (TY + WS_PW) * 32;
constexpr int AXW = TX + 2, AYW = TY + 2;    // aux tile: columns i0-1..i0+TX, rows j0-1..j0+TY
constexpr int A_SLOT = AXW * AYW;            // double2 per aux slot
#ifndef SAFARA_WS_PREG
#define SAFARA_WS_PREG 32                    // producer registers after setmaxnreg.dec
#endif
// consumer registers after setmaxnreg.inc: the rest of the 64K register file
constexpr int WS_CREG = ((65536 / 32 - WS_PW * SAFARA_WS_PREG) / TY) / 8 * 8;
static_assert(WS_CREG >= 128 && WS_CREG <= 256, "consumer register budget");

// Shared memory: a u ring of WS_US plane tiles (with halo 2), the aux ring
// (one (rho_i, square) tile per u slot) and a separate, shallower forcing ring
// of WS_FS slots -- forcing(k) is read only at step k, u(k) already at step
// k-2 (own column), so splitting the rings buys one more u plane of TMA
// lookahead in the same shared memory.
#ifndef SAFARA_WS_US
#define SAFARA_WS_US 4
#endif
#ifndef SAFARA_WS_FS
#define SAFARA_WS_FS 2
#endif
constexpr int WS_US = SAFARA_WS_US, WS_FS = SAFARA_WS_FS;
constexpr size_t WS_U_BYTES = (size_t)WS_US * U_SLOT * 8;
// (padded: the forcing ring behind it is a TMA destination, 128-byte aligned)
constexpr size_t WS_AUX_BYTES = ((size_t)WS_US * A_SLOT * 16 + 127) / 128 * 128;
constexpr size_t WS_F_BYTES = (size_t)WS_FS * F_SLOT * 8;
constexpr size_t WS_BAR_OFF = WS_U_BYTES + WS_AUX_BYTES + WS_F_BYTES;
constexpr size_t WS_SMEM_BYTES = WS_BAR_OFF + (3 * WS_US + 2 * WS_FS) * 8;
static_assert(WS_SMEM_BYTES <= 227 * 1024, "WS shared memory");
static_assert(WS_U_BYTES % 128 == 0 && (U_SLOT * 8) % 128 == 0 && (F_SLOT * 8) % 128 == 0 &&
                  (WS_U_BYTES + WS_AUX_BYTES) % 128 == 0,
              "TMA destinations 128-byte aligned");


// Device-side coefficients: safara_coeffs_t plus the constant products that
// the NAS text evaluates left to right (xxcon2*con43 -> one double).
struct Coef {
    double dt, dssp, c1, c2;
    double t2[3];          // tx2, ty2, tz2
    double d1[3][5];       // dx{m}tx1, dy{m}ty1, dz{m}tz1
    double con2[3], con2x43[3], con3[3], con4[3], con5[3];
    double c1c2;           // c1*c2 (SP speed, aux output only)
};

struct Params {
    int nx, ny, nz;        // global extents
    int sy, sm, sk;        // shared element strides (dim clause), int32 (small)
    // ablation copies (SAFARA_INDEX 1/2 builds only; same values)
    int u_sy, u_sm, u_sk, f_sy, f_sm, f_sk, r_sy, r_sm, r_sk;
    long long u_sy64, u_sm64, u_sk64, f_sy64, f_sm64, f_sk64, r_sy64, r_sm64, r_sk64;
    int k0;                // global k of forcing/rhs local plane 0
    int ukoff;             // u local plane = k - k0 + ukoff
    int nzu;               // planes in the u buffer
    int ka0, kb0, ka1, kb1;// global planes to compute: [ka0,kb0) U [ka1,kb1)
    int n0, nplanes;       // n0 = kb0-ka0, nplanes = n0 + (kb1-ka1)
    int ntx, nty;          // column tiles
    int ncol;              // ntx * nty
    int chunk;             // planes per chunk of the chunk-major unit order
    int ncta;              // compute CTAs (the grid has ncta + nface_cta)
    int nface_cta;         // extra CTAs that only copy boundary faces (0: compute CTAs do it)
    int parts;             // lockstep: k-parts per column (CTA c -> tile c % ncol); 0 = ranges
    int split_bias;        // lockstep: planes the last k-part gives to the others (f2)
    int units;             // ncol*nplanes (column-plane work items, < 2^31)
    int fk_lo, fk_hi;      // local planes whose boundary faces this launch copies
    int iface_tiles;       // 1: the i-face columns of the marched planes [ka0, kb0), rows
                           // 1..ny-2, are written by the edge column tiles (warp-specialised
                           // kernel, from the forcing tile in shared memory); the face
                           // CTAs skip them
    int pos_j, pos_m, pos_k;  // tensor-map dimension holding j, m, k
    const double *u;       // u buffer base (local plane 0)
    const double *f;       // forcing base (local plane 0)
    double *r;             // rhs base (local plane 0)
    double *aux;           // SURVEY §8(f) f1 aux output (NULL: none); component c of
                           // local plane kl at i + sy*j + sm*c + ska*kl
    int naux;              // 6 (rho_i, us, vs, ws, square, qs) or 7 (+ SP speed)
    int ska;               // aux plane stride
    // SURVEY §8(f) f2 (fused peer halo).  Global planes [pk_lo, pk_hi) are
    // read from the local u buffer; a plane k < pk_lo comes from the lower
    // neighbour's slab at u_lo + sk*(k + lo_koff), k >= pk_hi from the upper
    // one at u_hi + sk*(k + hi_koff) (peer pointers over NVLink).  Single-GPU
    // and ghost-slab launches: pk_lo = -2^30, pk_hi = 2^30, no peers.
    int pk_lo, pk_hi;
    int lo_koff, hi_koff;
    const double *u_lo, *u_hi;
    // Cross-GPU synchronisation (epoch > 0): pflags = this rank's flag words
    // (SAFARA_PEER_* indices), pflags_lo / pflags_hi = the neighbours'.
    unsigned long long *pflags, *pflags_lo, *pflags_hi;
    unsigned long long epoch;  // 0: none; SAFARA_PEER_EPOCH_AUTO: device counter
    unsigned long long peer_timeout_ns;  // bounded flag waits, then __trap()
    double *norm_part;     // f1 fused rhs_norm: per-CTA partial sums [m * ncta + cta] (NULL: none)
    unsigned long long *norm_ctr;  // CTAs done (0 between passes; the last CTA resets it)
    double *norm_out;      // 5 doubles: sqrt(sum / norm_npts), or the sums if norm_npts == 0
    double norm_npts;
    unsigned long long *dbg;  // SAFARA_TIMELINE builds: per-CTA {start, end, smid}
    unsigned long long *steplog;  // SAFARA_STEPLOG builds: per-CTA globaltimer at each step
    Coef c;
};

// Launchers implemented in rhs_fast.cu / rhs_strict.cu.
// uniform_d: every d1[ax][0..4] equal (NAS: dx1..dx5 = 0.75 ...), which lets
// the kernel keep one d1 per axis in uniform registers.
cudaError_t launch_rhs_fast(const CUtensorMap &umap, const CUtensorMap &fmap, const Params &p,
                            bool uniform_d, cudaStream_t s);
cudaError_t launch_rhs_strict(const CUtensorMap &umap, const CUtensorMap &fmap, const Params &p,
                              bool uniform_d, cudaStream_t s);
// norm.cu: per-component sums of squares over interior points (f1)
int norm_grid();
// npts > 0: finish NPB rhs_norm in the same launch, out[m] = sqrt(sum/npts)
cudaError_t launch_sumsq(const double *rhs, int nx, int ny, int sy, int sm, int sk, int kl0, int nk,
                         double *work, double *out, cudaStream_t s, double npts = 0.0);
// v[m] = sqrt(v[m] / npts), m < 5 (rhs_norm after a cross-slab all-reduce)
cudaError_t launch_rms_finish(double *v, double npts, cudaStream_t s);
// f1 fused norm: out[m] = sum over the G per-CTA partials work[m * G + b]
// (in b order), sqrt(sum / npts) when npts > 0
cudaError_t launch_partials_final(const double *work, int G, double *out, double npts,
                                  cudaStream_t s);
// api.cu: the launch counter behind safara_launch_count
void count_launches(int n);

// seismic.cu: PAPER.md Fig. 8 dz loop (f4); the bulk-copy kernel when the
// rows are 16-byte aligned (SAFARA_SEISMIC_LDG=1 forces the LDG kernel)
cudaError_t launch_seismic_dz(const double *vz1, const double *vz2, const double *vz3, double *out,
                              int nx, int ny, int nz, int sy, int sk, double h, int sms,
                              cudaStream_t s);

// bt_solve.cu: SURVEY §8(f) f4(ii), the NPB BT line solves / add / error norm
int bt_work_doubles(int nx, int ny, int nz);
cudaError_t launch_bt_solve(int dir, const double *u, const double *aux, double *rhs,
                            double *work, int nx, int ny, int nz, int sy, int sm, int sk, int ska,
                            const safara_bt_coeffs_t &bc, cudaStream_t s);
cudaError_t launch_bt_add(double *u, const double *rhs, int nx, int ny, int nz, int sy, int sm,
                          int sk, int sms, cudaStream_t s);
int err_norm_grid();
cudaError_t launch_error_norm(const double *u, const double *ue, int nx, int ny, int nz, int sy,
                              int sm, int sk, double *work, double *rms, cudaStream_t s);

// Round 2: the warp-specialised kernels (rhs_ws.cuh; one segment per CTA, no
// aux output, no peer halo).  attr: 2 entries (uniform d1, general).
cudaError_t launch_rhs_ws_fast(const CUtensorMap &umap, const CUtensorMap &fmap, const Params &p,
                               bool uniform_d, cudaStream_t s);
cudaError_t launch_rhs_ws_strict(const CUtensorMap &umap, const CUtensorMap &fmap, const Params &p,
                                 bool uniform_d, cudaStream_t s);
cudaError_t setup_rhs_ws_fast(cudaFuncAttributes *attr);
cudaError_t setup_rhs_ws_strict(cudaFuncAttributes *attr);

// attr: 4 entries (production NAS path, general coefficients, aux, NAS + aux)
cudaError_t setup_rhs_fast(int *ctas_per_sm, cudaFuncAttributes *attr);
cudaError_t setup_rhs_strict(int *ctas_per_sm, cudaFuncAttributes *attr);

}  // namespace safara
