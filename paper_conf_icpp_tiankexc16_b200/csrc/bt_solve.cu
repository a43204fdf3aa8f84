// bt_solve.cu -- SURVEY §8(f) f4(ii): the rest of one NPB BT time step
// around compute_rhs, so that the library runs a whole BT step on the GPU
// and reproduces NPB's verification norms (include/safara.h safara_bt_*).
//
//   step = safara_rhs_aux (compute_rhs + the step-0 fields rho_i, qs, square
//          the Jacobians need) -> x_solve -> y_solve -> z_solve -> add
//
// Each solve is NPB's approximate-factorisation line solve (x_solve.f ...):
// for every interior grid line along the direction, the 5x5
// block-tridiagonal system  AA(l) x(l-1) + BB(l) x(l) + CC(l) x(l+1) = rhs(l)
// with AA = -dt t2 fjac(l-1) - dt t1 (njac(l-1) + d), BB = I + 2 dt t1
// (njac(l) + d), CC = dt t2 fjac(l+1) - dt t1 (njac(l+1) + d) (d = diag of
// dx1..dx5 for xi), identity end blocks (lhsinit), by block Gaussian
// elimination without pivoting (solve_subs.f binvcrhs / matvec_sub /
// matmul_sub) and back substitution, in place on rhs.
//
// Not the hot path (the compute_rhs pass is): a plain kernel, one thread per
// line marching along it (the sequential loop; SAFARA's split, PAPER.md
// L684-692), C' blocks in a global scratch laid out [l][25][line] so that the
// threads of a warp touch consecutive words.  Compiled with --fmad=false and
// written in NPB's operation order (the oracle's nas_bt.c order), so it is
// bit-identical to the oracle whenever its inputs are (STRICT rhs/aux).
#include <cstdint>

#include "safara_internal.h"

namespace safara {
namespace {

struct BtDev {
    double dt, c1, c2, c3c4, c1345, con43;
    double t1[3], t2[3];
    double d[3][5];
};

// u / rhs: canonical [k][m][j][i] (strides sy, sm, sk); aux: rho_i (0),
// square (4), qs (5) of (i, j, k) at i + sy*j + sm*c + ska*k.
struct Line {
    const double *u, *aux;
    double *rhs, *work;
    int nx, ny, nz, sy, sm, sk, ska;
    int nlines;
};

// Flux Jacobian fjac and viscous Jacobian njac at one point (x/y/z_solve.f),
// direction a = 1 (xi), 2 (eta), 3 (zeta) = 0-based index of the normal
// momentum.  Same expression trees as oracle/nas_bt.c jacobians().
__device__ void jacobians(int a, const BtDev &c, const double (&u)[5], double rho_i, double qs,
                          double square, double (&fjac)[5][5], double (&njac)[5][5]) {
    const double tmp1 = rho_i, tmp2 = tmp1 * tmp1, tmp3 = tmp1 * tmp2;
    const double c1 = c.c1, c2 = c.c2, c3c4 = c.c3c4, con43 = c.con43, c1345 = c.c1345;
#pragma unroll
    for (int r = 0; r < 5; ++r)
#pragma unroll
        for (int s = 0; s < 5; ++s) {
            fjac[r][s] = 0.0;
            njac[r][s] = 0.0;
        }
    fjac[0][a] = 1.0;
#pragma unroll
    for (int r = 1; r <= 3; ++r) {
        if (r == a) {
            fjac[r][0] = -(u[a] * u[a] * tmp2) + c2 * qs;
#pragma unroll
            for (int s = 1; s <= 3; ++s)
                fjac[r][s] = (s == a) ? (2.0 - c2) * (u[a] * tmp1) : -c2 * (u[s] * tmp1);
            fjac[r][4] = c2;
        } else {
            fjac[r][0] = -(u[r] * u[a]) * tmp2;
            fjac[r][a] = u[r] * tmp1;
            fjac[r][r] = u[a] * tmp1;
        }
    }
    fjac[4][0] = (c2 * 2.0 * square - c1 * u[4]) * (u[a] * tmp2);
#pragma unroll
    for (int s = 1; s <= 3; ++s)
        fjac[4][s] = (s == a) ? c1 * u[4] * tmp1 - c2 * (u[a] * u[a] * tmp2 + qs)
                              : -c2 * (u[s] * u[a]) * tmp2;
    fjac[4][4] = c1 * (u[a] * tmp1);
#pragma unroll
    for (int r = 1; r <= 3; ++r) {
        const double cr = (r == a) ? con43 * c3c4 : c3c4;
        njac[r][0] = -cr * tmp2 * u[r];
        njac[r][r] = cr * tmp1;
    }
    njac[4][0] = 0.0;
#pragma unroll
    for (int r = 1; r <= 3; ++r) {
        const double cr = (r == a) ? con43 * c3c4 : c3c4;
        njac[4][0] = njac[4][0] - (cr - c1345) * tmp3 * (u[r] * u[r]);
    }
    njac[4][0] = njac[4][0] - c1345 * tmp2 * u[4];
#pragma unroll
    for (int r = 1; r <= 3; ++r) {
        const double cr = (r == a) ? con43 * c3c4 : c3c4;
        njac[4][r] = (cr - c1345) * tmp2 * u[r];
    }
    njac[4][4] = c1345 * tmp1;
}

// Grid point l of this thread's line in direction DIR (element offset of
// (i, j, k) without the component / aux-component term).
template <int DIR>
__device__ __forceinline__ void coords(const Line &L, int line, int l, int &o, int &oa) {
    int i, j, k;
    if (DIR == 0) {        // lines (j, k), j fastest
        j = 1 + line % (L.ny - 2); k = 1 + line / (L.ny - 2); i = l;
    } else if (DIR == 1) { // lines (i, k), i fastest
        i = 1 + line % (L.nx - 2); k = 1 + line / (L.nx - 2); j = l;
    } else {               // lines (i, j), i fastest
        i = 1 + line % (L.nx - 2); j = 1 + line / (L.nx - 2); k = l;
    }
    o = i + L.sy * j + L.sk * k;
    oa = i + L.sy * j + L.ska * k;
}

template <int DIR>
__device__ void jac_at(const Line &L, const BtDev &c, int line, int l, double (&fj)[5][5],
                       double (&nj)[5][5]) {
    int o, oa;
    coords<DIR>(L, line, l, o, oa);
    double u[5];
#pragma unroll
    for (int m = 0; m < 5; ++m) u[m] = L.u[o + L.sm * m];
    const double rho = L.aux[oa], sq = L.aux[oa + 4 * L.sm], qs = L.aux[oa + 5 * L.sm];
    jacobians(DIR + 1, c, u, rho, qs, sq, fj, nj);
}

// solve_subs.f binvcrhs (C != nullptr) / binvrhs: Gauss-Jordan on lhs.
template <bool WITH_C>
__device__ void binvcrhs(double (&lhs)[5][5], double (&cb)[5][5], double (&r)[5]) {
#pragma unroll
    for (int p = 0; p < 5; ++p) {
        const double pivot = 1.00 / lhs[p][p];
#pragma unroll
        for (int n = p + 1; n < 5; ++n) lhs[p][n] = lhs[p][n] * pivot;
        if (WITH_C) {
#pragma unroll
            for (int n = 0; n < 5; ++n) cb[p][n] = cb[p][n] * pivot;
        }
        r[p] = r[p] * pivot;
#pragma unroll
        for (int q = 0; q < 5; ++q) {
            if (q == p) continue;
            const double coeff = lhs[q][p];
#pragma unroll
            for (int n = p + 1; n < 5; ++n) lhs[q][n] = lhs[q][n] - coeff * lhs[p][n];
            if (WITH_C) {
#pragma unroll
                for (int n = 0; n < 5; ++n) cb[q][n] = cb[q][n] - coeff * cb[p][n];
            }
            r[q] = r[q] - coeff * r[p];
        }
    }
}

template <int DIR>
__global__ void __launch_bounds__(128) bt_solve_kernel(Line L, BtDev c, int len) {
    const int line = blockIdx.x * blockDim.x + threadIdx.x;
    if (line >= L.nlines) return;
    const int isize = len - 1;
    const double dtt1 = c.dt * c.t1[DIR], dtt2 = c.dt * c.t2[DIR];
    double fprev[5][5], nprev[5][5], fcur[5][5], ncur[5][5], fnext[5][5], nnext[5][5];
    double cp[5][5];  // C' of the previous point
    double rp[5];     // r' of the previous point
    auto W = [&](int l, int e) -> double & {
        return L.work[((size_t)l * 25 + e) * L.nlines + line];
    };
    auto R = [&](int l, int m) -> double & {
        int o, oa;
        coords<DIR>(L, line, l, o, oa);
        (void)oa;
        return L.rhs[o + L.sm * m];
    };
    // l = 0: BB = I, CC = 0 (lhsinit) -> C'(0) = 0, r'(0) = r(0) exactly
#pragma unroll
    for (int m = 0; m < 5; ++m) {
        rp[m] = R(0, m);
#pragma unroll
        for (int n = 0; n < 5; ++n) {
            cp[m][n] = 0.0;
            W(0, m * 5 + n) = 0.0;
        }
    }
    jac_at<DIR>(L, c, line, 0, fprev, nprev);
    jac_at<DIR>(L, c, line, 1, fcur, ncur);
    for (int l = 1; l <= isize - 1; ++l) {
        jac_at<DIR>(L, c, line, l + 1, fnext, nnext);
        double aa[5][5], bb[5][5], cc[5][5];
#pragma unroll
        for (int r = 0; r < 5; ++r)
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                aa[r][s] = -dtt2 * fprev[r][s] - dtt1 * nprev[r][s];
                bb[r][s] = dtt1 * 2.0 * ncur[r][s];
                cc[r][s] = dtt2 * fnext[r][s] - dtt1 * nnext[r][s];
                if (r == s) {
                    aa[r][s] = aa[r][s] - dtt1 * c.d[DIR][r];
                    bb[r][s] = 1.0 + bb[r][s] + dtt1 * 2.0 * c.d[DIR][r];
                    cc[r][s] = cc[r][s] - dtt1 * c.d[DIR][r];
                }
            }
        double r[5];
#pragma unroll
        for (int m = 0; m < 5; ++m) r[m] = R(l, m);
        // matvec_sub: r = r - AA r'(l-1)
#pragma unroll
        for (int i = 0; i < 5; ++i)
            r[i] = r[i] - aa[i][0] * rp[0] - aa[i][1] * rp[1] - aa[i][2] * rp[2] -
                   aa[i][3] * rp[3] - aa[i][4] * rp[4];
        // matmul_sub: BB = BB - AA C'(l-1)
#pragma unroll
        for (int j = 0; j < 5; ++j)
#pragma unroll
            for (int i = 0; i < 5; ++i)
                bb[i][j] = bb[i][j] - aa[i][0] * cp[0][j] - aa[i][1] * cp[1][j] -
                           aa[i][2] * cp[2][j] - aa[i][3] * cp[3][j] - aa[i][4] * cp[4][j];
        binvcrhs<true>(bb, cc, r);
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            R(l, m) = r[m];
            rp[m] = r[m];
#pragma unroll
            for (int n = 0; n < 5; ++n) {
                cp[m][n] = cc[m][n];
                W(l, m * 5 + n) = cc[m][n];
            }
        }
#pragma unroll
        for (int r2 = 0; r2 < 5; ++r2)
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                fprev[r2][s] = fcur[r2][s];
                nprev[r2][s] = ncur[r2][s];
                fcur[r2][s] = fnext[r2][s];
                ncur[r2][s] = nnext[r2][s];
            }
    }
    // l = isize: AA = 0, BB = I (lhsinit): r(isize) is unchanged exactly
    double xn[5];
#pragma unroll
    for (int m = 0; m < 5; ++m) xn[m] = R(isize, m);
    // back substitution: r(l) = r(l) - C'(l) x(l+1)
    for (int l = isize - 1; l >= 0; --l) {
        double x[5];
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            double v = R(l, m);
#pragma unroll
            for (int n = 0; n < 5; ++n) v = v - W(l, m * 5 + n) * xn[n];
            x[m] = v;
        }
#pragma unroll
        for (int m = 0; m < 5; ++m) {
            R(l, m) = x[m];
            xn[m] = x[m];
        }
    }
}

// add.f: u = u + rhs on the interior points (one thread per (i, j, k, m)).
__global__ void bt_add_kernel(double *u, const double *rhs, int nx, int ny, int nz, int sy,
                              int sm, int sk) {
    const long long n = (long long)(nx - 2) * (ny - 2) * (nz - 2) * 5;
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < n;
         t += (long long)gridDim.x * blockDim.x) {
        const int i = 1 + (int)(t % (nx - 2));
        long long r = t / (nx - 2);
        const int j = 1 + (int)(r % (ny - 2));
        r /= (ny - 2);
        const int m = (int)(r % 5);
        const int k = 1 + (int)(r / 5);
        const int o = i + sy * j + sm * m + sk * k;
        u[o] = u[o] + rhs[o];
    }
}

constexpr int EN_THREADS = 256;

// error.f error_norm numerator, deterministic: block b of component m sums a
// fixed row range of ALL points; the finishing block sums the partials in
// block order and takes sqrt(sum / (nx-2) / (ny-2) / (nz-2)).
__global__ void __launch_bounds__(EN_THREADS)
err_partial(const double *u, const double *ue, int nx, int ny, int nz, int sy, int sm, int sk,
            double *work) {
    const int m = blockIdx.y, G = gridDim.x, b = blockIdx.x;
    const long long R = (long long)nz * ny;
    const long long r0 = R * b / G, r1 = R * (b + 1) / G;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    double acc = 0.0;
    for (long long r = r0 + warp; r < r1; r += EN_THREADS / 32) {
        const int k = (int)(r / ny), j = (int)(r % ny);
        const long long base = (long long)sy * j + (long long)sm * m + (long long)sk * k;
        for (int i = lane; i < nx; i += 32) {
            const double add = u[base + i] - ue[base + i];
            acc = acc + add * add;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_down_sync(0xffffffffu, acc, o);
    __shared__ double s[EN_THREADS / 32];
    if (lane == 0) s[warp] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < EN_THREADS / 32; ++w) t += s[w];
        work[m * G + b] = t;
    }
}

__global__ void err_final(const double *work, int G, int nx, int ny, int nz, double *rms) {
    const int m = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (m >= 5) return;
    double t = 0.0;
    for (int b = lane; b < G; b += 32) t += work[m * G + b];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) t += __shfl_down_sync(0xffffffffu, t, o);
    if (lane == 0) {
        t = t / (double)(nx - 2);
        t = t / (double)(ny - 2);
        t = t / (double)(nz - 2);
        rms[m] = sqrt(t);
    }
}

}  // namespace

int bt_work_doubles(int nx, int ny, int nz) {
    const long long a = (long long)(ny - 2) * (nz - 2) * nx, b = (long long)(nx - 2) * (nz - 2) * ny,
                    c = (long long)(nx - 2) * (ny - 2) * nz;
    long long m = a > b ? a : b;
    m = m > c ? m : c;
    m *= 25;
    return m >= (1LL << 31) ? -1 : (int)m;
}

cudaError_t launch_bt_solve(int dir, const double *u, const double *aux, double *rhs,
                            double *work, int nx, int ny, int nz, int sy, int sm, int sk, int ska,
                            const safara_bt_coeffs_t &bc, cudaStream_t s) {
    Line L;
    L.u = u; L.aux = aux; L.rhs = rhs; L.work = work;
    L.nx = nx; L.ny = ny; L.nz = nz; L.sy = sy; L.sm = sm; L.sk = sk; L.ska = ska;
    const int len = dir == 0 ? nx : dir == 1 ? ny : nz;
    L.nlines = dir == 0 ? (ny - 2) * (nz - 2) : dir == 1 ? (nx - 2) * (nz - 2) : (nx - 2) * (ny - 2);
    BtDev c;
    c.dt = bc.dt; c.c1 = bc.c1; c.c2 = bc.c2; c.c3c4 = bc.c3c4; c.c1345 = bc.c1c5 * bc.c3c4;
    c.con43 = bc.con43;
    c.t1[0] = bc.tx1; c.t1[1] = bc.ty1; c.t1[2] = bc.tz1;
    c.t2[0] = bc.tx2; c.t2[1] = bc.ty2; c.t2[2] = bc.tz2;
    for (int m = 0; m < 5; ++m) {
        c.d[0][m] = bc.dx[m];
        c.d[1][m] = bc.dy[m];
        c.d[2][m] = bc.dz[m];
    }
    const int T = 128, G = (L.nlines + T - 1) / T;
    if (dir == 0) bt_solve_kernel<0><<<G, T, 0, s>>>(L, c, len);
    else if (dir == 1) bt_solve_kernel<1><<<G, T, 0, s>>>(L, c, len);
    else bt_solve_kernel<2><<<G, T, 0, s>>>(L, c, len);
    return cudaGetLastError();
}

cudaError_t launch_bt_add(double *u, const double *rhs, int nx, int ny, int nz, int sy, int sm,
                          int sk, int sms, cudaStream_t s) {
    bt_add_kernel<<<sms * 4, 256, 0, s>>>(u, rhs, nx, ny, nz, sy, sm, sk);
    return cudaGetLastError();
}

int err_norm_grid() { return 148; }

cudaError_t launch_error_norm(const double *u, const double *ue, int nx, int ny, int nz, int sy,
                              int sm, int sk, double *work, double *rms, cudaStream_t s) {
    const int G = err_norm_grid();
    err_partial<<<dim3(G, 5), EN_THREADS, 0, s>>>(u, ue, nx, ny, nz, sy, sm, sk, work);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    err_final<<<1, 5 * 32, 0, s>>>(work, G, nx, ny, nz, rms);
    return cudaGetLastError();
}

}  // namespace safara

// ---- C ABI (include/safara.h) ------------------------
namespace {

bool canonical_like(const safara_dims_t *d) {
    // j second-fastest, components inside a plane: the [k][m][j][i] order
    return d && d->sm >= d->sy * d->ny && d->sk >= 5 * d->sm;
}

int aux_stride(const safara_dims_t *d) { return 6 * d->sm; }

bool overlap(const void *a, long long an, const void *b, long long bn) {
    const uintptr_t a0 = (uintptr_t)a, b0 = (uintptr_t)b;
    return a0 < b0 + (uintptr_t)bn && b0 < a0 + (uintptr_t)an;
}

int check_solve_args(const double *u, const double *aux, const double *rhs, const double *work,
                     const safara_dims_t *dims) {
    if (!u || !aux || !rhs || !work || !dims) return SAFARA_ERR_ARG;
    int rc = safara_validate_dims(dims, dims->nz);
    if (rc) return rc;
    if (!canonical_like(dims)) return SAFARA_ERR_LAYOUT;
    if (((uintptr_t)u | (uintptr_t)aux | (uintptr_t)rhs | (uintptr_t)work) & 7u)
        return SAFARA_ERR_ALIGN;
    const long long ab = ((long long)aux_stride(dims) * dims->nz) * 8;
    if ((long long)aux_stride(dims) * dims->nz >= (1LL << 31)) return SAFARA_ERR_TOO_LARGE;
    const long long fb = ((long long)dims->sk * dims->nz) * 8;
    const int wd = safara::bt_work_doubles(dims->nx, dims->ny, dims->nz);
    if (wd < 0) return SAFARA_ERR_TOO_LARGE;
    const long long wb = (long long)wd * 8;
    if (overlap(rhs, fb, u, fb) || overlap(rhs, fb, aux, ab) || overlap(work, wb, rhs, fb) ||
        overlap(work, wb, u, fb) || overlap(work, wb, aux, ab))
        return SAFARA_ERR_ARG;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return SAFARA_ERR_CUDA;
    return SAFARA_OK;
}

}  // namespace

extern "C" {

int safara_bt_coeffs_nas(int nx, int ny, int nz, double dt, safara_bt_coeffs_t *out) {
    if (!out) return SAFARA_ERR_ARG;
    if (nx < 2 || ny < 2 || nz < 2) return SAFARA_ERR_SHAPE;
    // NPB set_constants.f: the values the solves use
    const double c1 = 1.4, c2 = 0.4, c3 = 0.1, c4 = 1.0, c5 = 1.4;
    const double dnxm1 = 1.0 / (double)(nx - 1), dnym1 = 1.0 / (double)(ny - 1),
                 dnzm1 = 1.0 / (double)(nz - 1);
    out->dt = dt;
    out->c1 = c1;
    out->c2 = c2;
    out->c3c4 = c3 * c4;
    out->c1c5 = c1 * c5;
    out->con43 = 4.0 / 3.0;
    out->tx1 = 1.0 / (dnxm1 * dnxm1);
    out->tx2 = 1.0 / (2.0 * dnxm1);
    out->ty1 = 1.0 / (dnym1 * dnym1);
    out->ty2 = 1.0 / (2.0 * dnym1);
    out->tz1 = 1.0 / (dnzm1 * dnzm1);
    out->tz2 = 1.0 / (2.0 * dnzm1);
    for (int m = 0; m < 5; ++m) {
        out->dx[m] = 0.75;
        out->dy[m] = 0.75;
        out->dz[m] = 1.0;
    }
    return SAFARA_OK;
}

int safara_bt_work_doubles(int nx, int ny, int nz) {
    if (nx < 6 || ny < 6 || nz < 6) return SAFARA_ERR_SHAPE;
    const int w = safara::bt_work_doubles(nx, ny, nz);
    return w < 0 ? SAFARA_ERR_TOO_LARGE : w;
}

int safara_bt_solve(int dir, const double *u, const double *aux, double *rhs, double *work,
                    const safara_dims_t *dims, const safara_bt_coeffs_t *bc, void *stream) {
    if (dir < 0 || dir > 2 || !bc) return SAFARA_ERR_ARG;
    int rc = check_solve_args(u, aux, rhs, work, dims);
    if (rc) return rc;
    cudaError_t e = safara::launch_bt_solve(dir, u, aux, rhs, work, dims->nx, dims->ny, dims->nz,
                                            dims->sy, dims->sm, dims->sk, aux_stride(dims), *bc,
                                            (cudaStream_t)stream);
    if (e != cudaSuccess) return SAFARA_ERR_CUDA;
    safara::count_launches(1);
    return SAFARA_OK;
}

int safara_bt_add(double *u, const double *rhs, const safara_dims_t *dims, void *stream) {
    if (!u || !rhs || !dims) return SAFARA_ERR_ARG;
    int rc = safara_validate_dims(dims, dims->nz);
    if (rc) return rc;
    if (((uintptr_t)u | (uintptr_t)rhs) & 7u) return SAFARA_ERR_ALIGN;
    const long long fb = ((long long)dims->sk * dims->nz) * 8;
    if (overlap(u, fb, rhs, fb)) return SAFARA_ERR_ARG;
    int dev = 0, sms = 0;
    if (cudaGetDevice(&dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
        return SAFARA_ERR_CUDA;
    cudaError_t e = safara::launch_bt_add(u, rhs, dims->nx, dims->ny, dims->nz, dims->sy, dims->sm,
                                          dims->sk, sms, (cudaStream_t)stream);
    if (e != cudaSuccess) return SAFARA_ERR_CUDA;
    safara::count_launches(1);
    return SAFARA_OK;
}

int safara_bt_step(double *u, const double *forcing, double *rhs, double *aux, double *work,
                   const safara_dims_t *dims, const safara_coeffs_t *coeffs,
                   const safara_bt_coeffs_t *bc, int flags, void *stream) {
    if (!bc || !coeffs) return SAFARA_ERR_ARG;
    int rc = check_solve_args(u, aux, rhs, work, dims);
    if (rc) return rc;
    rc = safara_rhs_aux(u, forcing, rhs, aux, SAFARA_AUX_BT, dims, coeffs, flags, stream);
    if (rc) return rc;
    for (int dir = 0; dir < 3; ++dir) {
        rc = safara_bt_solve(dir, u, aux, rhs, work, dims, bc, stream);
        if (rc) return rc;
    }
    return safara_bt_add(u, rhs, dims, stream);
}

int safara_error_norm(const double *u, const double *u_exact, const safara_dims_t *dims,
                      double *work, double *rms, void *stream) {
    if (!u || !u_exact || !dims || !work || !rms) return SAFARA_ERR_ARG;
    int rc = safara_validate_dims(dims, dims->nz);
    if (rc) return rc;
    if (((uintptr_t)u | (uintptr_t)u_exact | (uintptr_t)work | (uintptr_t)rms) & 7u)
        return SAFARA_ERR_ALIGN;
    if (safara_norm_work_doubles() < 5 * safara::err_norm_grid()) return SAFARA_ERR_ARG;
    cudaError_t e = safara::launch_error_norm(u, u_exact, dims->nx, dims->ny, dims->nz, dims->sy,
                                              dims->sm, dims->sk, work, rms, (cudaStream_t)stream);
    if (e != cudaSuccess) return SAFARA_ERR_CUDA;
    safara::count_launches(2);
    return SAFARA_OK;
}

}  // extern "C"
