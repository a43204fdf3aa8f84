"""P3: the oracle against the EXACT result, on tiny grids.

Every fp64 input and every fp64 constant of NPB set_constants is a dyadic
rational, so the operator of SURVEY App. A can be evaluated exactly with
``fractions.Fraction``.  The evaluation here is written independently of the
oracle's NAS line-by-line loop nest: per point and per axis in conservation
form -- Euler flux vector F(u) differenced centrally, second differences of
u, of the velocities, of qs, of the axis velocity squared and of u5*rho_i,
and the fourth-order dissipation from a 5-case weight table indexed by the
GLOBAL position along the axis -- with all the arithmetic exact, so the
evaluation order is immaterial.  The oracle (fp64, NAS order) must then sit
within a small fraction of the tolerance bound 1e-12 |x| + 1e-14 of the
exact value x at every point: a dropped term, a wrong sign, coefficient,
axis or stencil case shows up as an O(1) relative error instead.

Grids 6^3, 7^3 (the first size with all five dissipation cases distinct,
reading c4) and 9x8x7, inputs from nasgen (exact solution x (1 + 1e-3
noise), forcing = exact_rhs + noise).
"""
from fractions import Fraction as Fr

import numpy as np
import pytest

import nasgen
import oracle

RTOL, ATOL = 1e-12, 1e-14


def _diss_weights(x, n):
    """Weights of a[x-2..x+2] in NAS's 5-case fourth-order dissipation."""
    if x == 1:
        return (0, 0, 5, -4, 1)
    if x == 2:
        return (0, -4, 6, -4, 1)
    if x == n - 3:
        return (1, -4, 6, -4, 0)
    if x == n - 2:
        return (1, -4, 5, 0, 0)
    return (1, -4, 6, -4, 1)


def exact_rhs_pass(u, f, cs):
    """Exact App. A operator.  u, f: (nz, ny, nx, 5) float64 -> Fraction array."""
    nz, ny, nx, _ = u.shape
    C = {k: Fr(v) for k, v in cs.as_dict().items()}
    ext = (nx, ny, nz)
    d1 = [[C[f"d{a}{m}t{a}1"] for m in range(1, 6)] for a in "xyz"]
    t2 = [C["tx2"], C["ty2"], C["tz2"]]
    con = [[C[f"{a}{a}con{m}"] for m in range(1, 6)] for a in "xyz"]
    c1, c2, con43, dssp, dt = C["c1"], C["c2"], C["con43"], C["dssp"], C["dt"]

    U = {}

    def q(k, j, i):
        """Per-point exact quantities of point (i, j, k)."""
        key = (k, j, i)
        if key not in U:
            w = [Fr(float(x)) for x in u[k, j, i]]
            rho = 1 / w[0]
            vel = [w[1] * rho, w[2] * rho, w[3] * rho]
            sq = (w[1] ** 2 + w[2] ** 2 + w[3] ** 2) * rho / 2
            U[key] = (w, rho, vel, sq)
        return U[key]

    def flux(pt, a):
        """Euler flux vector along axis a (App. A steps 2/4/6, tx2 terms)."""
        w, rho, vel, sq = q(*pt)
        F = [w[1 + a]]
        for n in range(3):
            F.append(w[1 + n] * vel[a] + ((w[4] - sq) * c2 if n == a else 0))
        F.append((c1 * w[4] - c2 * sq) * vel[a])
        return F

    def smooth(pt, a):
        """The second-difference operands along axis a: u_m, vel_n, qs,
        vel_a^2, u5*rho_i."""
        w, rho, vel, sq = q(*pt)
        return w, vel, sq * rho, vel[a] ** 2, w[4] * rho

    out = np.empty((nz, ny, nx, 5), dtype=object)
    for k in range(nz):
        for j in range(ny):
            for i in range(nx):
                fr = [Fr(float(x)) for x in f[k, j, i]]
                if i in (0, nx - 1) or j in (0, ny - 1) or k in (0, nz - 1):
                    out[k, j, i] = fr            # boundary faces: rhs = forcing
                    continue
                r = list(fr)
                pos = (i, j, k)
                for a in range(3):
                    def at(s, a=a):
                        p = list(pos)
                        p[a] += s
                        return (p[2], p[1], p[0])
                    Fp, Fq = flux(at(1), a), flux(at(-1), a)
                    Sp, S0, Sq = smooth(at(1), a), smooth(at(0), a), smooth(at(-1), a)

                    def d2(idx, sub=None):
                        g = (lambda s: s[idx]) if sub is None else (lambda s: s[idx][sub])
                        return g(Sp) - 2 * g(S0) + g(Sq)

                    for m in range(5):
                        r[m] += d1[a][m] * d2(0, m) - t2[a] * (Fp[m] - Fq[m])
                    for n in range(3):
                        r[1 + n] += con[a][1] * (con43 if n == a else 1) * d2(1, n)
                    r[4] += con[a][2] * d2(2) + con[a][3] * d2(3) + con[a][4] * d2(4)
                    wts = _diss_weights(pos[a], ext[a])
                    for m in range(5):
                        r[m] -= dssp * sum(wt * q(*at(s))[0][m]
                                           for s, wt in zip(range(-2, 3), wts) if wt)
                out[k, j, i] = [x * dt for x in r]
    return out


@pytest.mark.parametrize("shape", [(6, 6, 6), (7, 7, 7), (7, 8, 9)])
def test_p3_oracle_within_bound_of_exact(shape):
    nz, ny, nx = shape
    inp = nasgen.make_inputs(nx, ny, nz, seed=11, A=1e-3, B=1e-2, dt=0.01)
    cs = oracle.set_constants(nx, ny, nz, inp.dt)
    o = oracle.compute_rhs(inp.u, inp.forcing, consts=cs)
    x = exact_rhs_pass(inp.u, inp.forcing, cs)
    worst = 0.0
    for idx in np.ndindex(nz, ny, nx):
        for m in range(5):
            ex = x[idx][m]
            err = abs(Fr(float(o[idx + (m,)])) - ex)
            bound = Fr(RTOL) * abs(ex) + Fr(ATOL)
            worst = max(worst, float(err / bound))
    # fp64 rounding in NAS order only: a small fraction of the bound
    assert worst < 0.05, worst


def test_p3_detects_a_flipped_sign():
    """The pin is sharp: negating one momentum flux term in the exact
    evaluation moves it far outside the bound."""
    nz = ny = nx = 7
    inp = nasgen.make_inputs(nx, ny, nz, seed=12, B=1e-2, dt=0.01)
    cs = oracle.set_constants(nx, ny, nz, inp.dt)
    o = oracle.compute_rhs(inp.u, inp.forcing, consts=cs)
    u2 = inp.u.copy()
    u2[:, :, :, 2] *= -1.0           # flips vs's sign -> different operator value
    x = exact_rhs_pass(u2, inp.forcing, cs)
    ratio = max(abs(float(Fr(float(o[3, 3, 3, m])) - x[3, 3, 3][m])) /
                (RTOL * abs(float(x[3, 3, 3][m])) + ATOL) for m in range(5))
    assert ratio > 1e3
