/*
 * oracle/nas_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * The CPU oracle for one NAS BT/SP `compute_rhs` pass: the loop nest whose
 * SAFARA / dim / small optimisation the paper evaluates (PAPER.md L1330-1362,
 * L1470-1488: "BT, LU and SP have several kernels that contain uncoalesced
 * memory accesses"; NPB-OpenACC suite [20], L2020-2023).  The paper itself never
 * writes the loop nest down; the definition transcribed here is NPB 3.x
 * rhs.f / set_constants.f as recalled in SURVEY.md Appendix A/B (reading c1,
 * c2 in DESIGN.md).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  It shares no code, header, constant
 * table or helper with the CUDA path under paper_conf_icpp_tiankexc16_b200/.
 *
 * Layout: NAS-BT C layout  u[nz][ny'][nx'][5]  with nx' = (nx/2)*2+1,
 * ny' = (ny/2)*2+1 (the NPB "IMAXP+1" padding).  Deliberately different from
 * the GPU layout so that layout marshalling is exercised by every parity test.
 *
 * Parity pins (tests/test_oracle_pins.py): P1 constant field closed form,
 * P2 exact-solution residual against the independently formulated
 * nasgen.exact_rhs, P3 exact-rational brute force, P4 polynomial / impulse
 * closed forms (dissipation operator = B^T B), P5 forcing affinity, P6 i<->j
 * symmetry, P7 O(h^2) convergence to the compressible Navier-Stokes operator
 * (tests/test_oracle_euler_pins.py: pins c1, c2, t?2 and the viscous /
 * artificial-dissipation constant combinations), P8 NPB verification
 * (tests/test_oracle_bt_pins.py): the full BT time step of nas_bt.c from NPB's
 * initialize reproduces NPB BT's own class S/W/A verification norms to
 * <= 1e-12 (NPB accepts 1e-8), which pins the physical parameter values
 * (gamma, mu, Pr, dx..dz, dssp) against NPB itself (reading c2).
 */
#ifndef NAS_ORACLE_H
#define NAS_ORACLE_H

typedef struct {
    double dt;
    double c1, c2, c3, c4, c5;
    double c1c2, c1c5, c3c4, conz1, con43, con16;
    double dnxm1, dnym1, dnzm1;
    double tx1, tx2, tx3, ty1, ty2, ty3, tz1, tz2, tz3;
    double dx1, dx2, dx3, dx4, dx5;
    double dy1, dy2, dy3, dy4, dy5;
    double dz1, dz2, dz3, dz4, dz5;
    double dssp;
    double dx1tx1, dx2tx1, dx3tx1, dx4tx1, dx5tx1;
    double dy1ty1, dy2ty1, dy3ty1, dy4ty1, dy5ty1;
    double dz1tz1, dz2tz1, dz3tz1, dz4tz1, dz5tz1;
    double c3c4tx3, c3c4ty3, c3c4tz3;
    double xxcon1, xxcon2, xxcon3, xxcon4, xxcon5;
    double yycon1, yycon2, yycon3, yycon4, yycon5;
    double zzcon1, zzcon2, zzcon3, zzcon4, zzcon5;
} oracle_consts_t;

/* NPB set_constants.f subset.  Returns 0, or -1 if any n < 2. */
int oracle_set_constants(int nx, int ny, int nz, double dt, oracle_consts_t *c);

/* Padded leading dimension used by the NAS-BT layout. */
int oracle_padded(int n);

/* One compute_rhs pass in NAS-BT layout.
 * u, forcing, rhs: nz*ny'*nx'*5 doubles each, caller-owned, no aliasing.
 * nthreads: OpenMP threads over k (result is identical for any count).
 * Returns 0, or -1 if any extent < 6 (reading c4: the 5-case dissipation
 * overlaps at n = 5 and reads outside the grid below that). */
int oracle_compute_rhs(int nx, int ny, int nz, const oracle_consts_t *c,
                       const double *u, const double *forcing, double *rhs,
                       int nthreads);

/* NAS step 0 auxiliary fields at every point: naux = 6
 * (rho_i, us, vs, ws, square, qs, the BT rhs.f order) or 7 (+ SP speed).
 * aux: [nz][ny'][nx'][naux].  Returns 0 or -1 on bad arguments. */
int oracle_compute_aux(int nx, int ny, int nz, const oracle_consts_t *c,
                       const double *u, double *aux, int naux);

/* NPB error.f rhs_norm numerator: out[m] = sum over interior points of
 * rhs(m)^2 (k, j, i loop order).  Returns 0 or -1. */
int oracle_rhs_sumsq(int nx, int ny, int nz, const double *rhs, double *out);

/* 355.seismic dz loop of PAPER.md Fig. 8 (zero lower bounds; see .c).
 * Dense Fortran-order arrays vz(i,j,k) at i + nx*(j + ny*k).  Returns 0/-1. */
int oracle_seismic_dz(int nx, int ny, int nz, const double *vz_1, const double *vz_2,
                      const double *vz_3, double *value_dz, double h);

/* ---- the rest of an NPB BT time step (nas_bt.c) ----
 * oracle_bt_solve: x_solve (dir 0), y_solve (1) or z_solve (2) of NPB BT:
 *   for every interior line, the 5x5 block-tridiagonal system of the
 *   approximate factorisation, solved in place on rhs (NAS layout); aux =
 *   oracle_compute_aux(naux = 6) of u.  Returns 0 / -1.
 * oracle_bt_add: u += rhs at interior points (add.f).
 * oracle_bt_run: niter NPB adi steps (compute_rhs, x/y/z_solve, add) on u in
 *   place; rhs (5/pt) and aux (6/pt) are caller scratch in NAS layout.
 * oracle_error_norm: NPB error_norm of u against u_exact (both NAS layout). */
int oracle_bt_solve(int dir, int nx, int ny, int nz, const oracle_consts_t *c,
                    const double *u, const double *aux, double *rhs);
int oracle_bt_add(int nx, int ny, int nz, double *u, const double *rhs);
int oracle_bt_run(int nx, int ny, int nz, const oracle_consts_t *c, double *u,
                  const double *forcing, double *rhs, double *aux, int niter,
                  int nthreads);
int oracle_error_norm(int nx, int ny, int nz, const double *u, const double *u_exact,
                      double *rms);

#endif
