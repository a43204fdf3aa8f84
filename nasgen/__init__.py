"""Seeded synthetic inputs for the NAS BT/SP ``compute_rhs`` pass.

This module is the ONLY code shared by the oracle side (``oracle/``, tests) and
the CUDA side (``paper_conf_icpp_tiankexc16_b200``, bench).  It holds none of
the hot path's arithmetic: it produces ``u`` and ``forcing`` the way the NPB
benchmark initialises them (NPB ``exact_solution.f`` / ``exact_rhs.f`` as
recalled in SURVEY.md App. B; the paper runs NPB-ACC class C, PAPER.md
L1354-1362), plus seeded relative noise (reading c11):

    u       = exact_solution(i/(nx-1), j/(ny-1), k/(nz-1)) * (1 + A * xi)
    forcing = exact_rhs(nx, ny, nz) + B * xi'

``xi, xi'`` in [-1, 1) come from a counter-based splitmix64 of
(seed, stream, linear index), so any sub-block can be regenerated
independently.  ``exact_rhs`` is NPB's own forcing generator: a *different
formulation* of the same discrete operator (buf/cuf/q arrays, xxcon1 and
0.5*xxcon3 instead of xxcon2*con43 and d2(qs)), which is why
``compute_rhs(exact_solution, exact_rhs) ~ 0`` is an independent pin (P2).

Arrays are returned in the logical layout ``(nz, ny, nx, 5)`` float64, C order.
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np

# NPB problem classes used by BASELINE.json (n, dt); SURVEY App. B table.
CLASSES = {
    ("BT", "S"): (12, 0.010),
    ("BT", "W"): (24, 0.0008),
    ("BT", "A"): (64, 0.0008),
    ("BT", "B"): (102, 0.0003),
    ("BT", "C"): (162, 0.0001),
    ("SP", "S"): (12, 0.015),
    ("SP", "W"): (36, 0.0015),
    ("SP", "A"): (64, 0.0015),
    ("SP", "B"): (102, 0.001),
    ("SP", "C"): (162, 0.00067),
}

# BASELINE.json configs, in order (configs[0] .. configs[4]).
CONFIGS = [("BT", "S"), ("SP", "W"), ("BT", "A"), ("SP", "B"), ("BT", "C")]

# NPB exact_solution coefficients ce(m, 1..13), m = 1..5.
CE = np.array([
    [2.0, 0.0, 0.0, 4.0, 5.0, 3.0, 0.5, 0.02, 0.01, 0.03, 0.5, 0.4, 0.3],
    [1.0, 0.0, 0.0, 0.0, 1.0, 2.0, 3.0, 0.01, 0.03, 0.02, 0.4, 0.3, 0.5],
    [2.0, 2.0, 0.0, 0.0, 0.0, 2.0, 3.0, 0.04, 0.03, 0.05, 0.3, 0.5, 0.4],
    [2.0, 2.0, 0.0, 0.0, 0.0, 2.0, 3.0, 0.03, 0.05, 0.04, 0.2, 0.1, 0.3],
    [5.0, 4.0, 3.0, 2.0, 0.1, 0.4, 0.3, 0.05, 0.04, 0.03, 0.1, 0.3, 0.2],
])


@dataclass(frozen=True)
class GenConsts:
    """The NPB set_constants values exact_rhs needs (generator's own copy)."""
    nx: int
    ny: int
    nz: int
    dt: float

    def __post_init__(self):
        c1, c2, c3, c4, c5 = 1.4, 0.4, 0.1, 1.0, 1.4
        d = {}
        d["c1"], d["c2"] = c1, c2
        dnxm1, dnym1, dnzm1 = 1.0 / (self.nx - 1), 1.0 / (self.ny - 1), 1.0 / (self.nz - 1)
        d["dnxm1"], d["dnym1"], d["dnzm1"] = dnxm1, dnym1, dnzm1
        c1c5 = c1 * c5
        c3c4 = c3 * c4
        tx1, tx2, tx3 = 1.0 / (dnxm1 * dnxm1), 1.0 / (2.0 * dnxm1), 1.0 / dnxm1
        ty1, ty2, ty3 = 1.0 / (dnym1 * dnym1), 1.0 / (2.0 * dnym1), 1.0 / dnym1
        tz1, tz2, tz3 = 1.0 / (dnzm1 * dnzm1), 1.0 / (2.0 * dnzm1), 1.0 / dnzm1
        d["tx2"], d["ty2"], d["tz2"] = tx2, ty2, tz2
        dx, dy, dz = 0.75, 0.75, 1.0
        d["dssp"] = 0.25 * max(dx, max(dy, dz))
        d["dxt"] = dx * tx1
        d["dyt"] = dy * ty1
        d["dzt"] = dz * tz1
        conz1, con43, con16 = 1.0 - c1c5, 4.0 / 3.0, 1.0 / 6.0
        for ax, t3 in (("xx", tx3), ("yy", ty3), ("zz", tz3)):
            c34 = c3c4 * t3
            d[ax + "con1"] = c34 * con43 * t3
            d[ax + "con2"] = c34 * t3
            d[ax + "con3"] = c34 * conz1 * t3
            d[ax + "con4"] = c34 * con16 * t3
            d[ax + "con5"] = c34 * c1c5 * t3
        object.__setattr__(self, "_d", d)

    def __getattr__(self, name):
        d = object.__getattribute__(self, "_d")
        if name in d:
            return d[name]
        raise AttributeError(name)


# ----------------------------------------------------------------------------
# Counter-based noise (splitmix64 finaliser over (seed, stream, index)).
# ----------------------------------------------------------------------------
_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 output function applied elementwise to uint64 counters."""
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)) & _M64
        z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & _M64
        z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & _M64
        return z ^ (z >> np.uint64(31))


def uniform_pm1(seed: int, stream: int, shape) -> np.ndarray:
    """Deterministic xi in [-1, 1) for every element of ``shape`` (C order)."""
    n = int(np.prod(shape))
    idx = np.arange(n, dtype=np.uint64)
    key = np.uint64(((seed & 0xFFFFF) << 44) | ((stream & 0xF) << 40))
    z = splitmix64(idx ^ key)
    x = (z >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    return (2.0 * x - 1.0).reshape(shape)


# ----------------------------------------------------------------------------
# NPB exact_solution / exact_rhs.
# ----------------------------------------------------------------------------
def exact_solution(xi, eta, zeta) -> np.ndarray:
    """NPB exact_solution on broadcastable coordinate arrays; last axis = m."""
    xi, eta, zeta = np.broadcast_arrays(*(np.asarray(a, dtype=np.float64) for a in (xi, eta, zeta)))
    out = np.empty(xi.shape + (5,), dtype=np.float64)
    for m in range(5):
        ce = CE[m]
        out[..., m] = (ce[0]
                       + xi * (ce[1] + xi * (ce[4] + xi * (ce[7] + xi * ce[10])))
                       + eta * (ce[2] + eta * (ce[5] + eta * (ce[8] + eta * ce[11])))
                       + zeta * (ce[3] + zeta * (ce[6] + zeta * (ce[9] + zeta * ce[12]))))
    return out


def exact_grid(nx: int, ny: int, nz: int) -> np.ndarray:
    """exact_solution at every grid point, shape (nz, ny, nx, 5)."""
    xi = np.arange(nx, dtype=np.float64) * (1.0 / (nx - 1))
    eta = np.arange(ny, dtype=np.float64) * (1.0 / (ny - 1))
    zeta = np.arange(nz, dtype=np.float64) * (1.0 / (nz - 1))
    return exact_solution(xi[None, None, :], eta[None, :, None], zeta[:, None, None])


def nas_initialize(nx: int, ny: int, nz: int) -> np.ndarray:
    """NPB initialize.f: the starting u of a BT/SP run, shape (nz, ny, nx, 5).

    Interior: transfinite (trilinear-blended) interpolation of the six faces'
    exact solutions, Pxi + Peta + Pzeta - Pxi*Peta - Pxi*Pzeta - Peta*Pzeta +
    Pxi*Peta*Pzeta with Pxi = xi*E(1,eta,zeta) + (1-xi)*E(0,eta,zeta) etc.;
    then the exact solution on the six boundary faces (input generation for
    the f4(ii) full-step check)."""
    dn = (1.0 / (nx - 1), 1.0 / (ny - 1), 1.0 / (nz - 1))
    xi = (np.arange(nx, dtype=np.float64) * dn[0])[None, None, :, None]
    eta = (np.arange(ny, dtype=np.float64) * dn[1])[None, :, None, None]
    zeta = (np.arange(nz, dtype=np.float64) * dn[2])[:, None, None, None]
    X, E, Z = (np.arange(nx) * dn[0])[None, None, :], (np.arange(ny) * dn[1])[None, :, None], \
        (np.arange(nz) * dn[2])[:, None, None]
    px0, px1 = exact_solution(0.0, E, Z), exact_solution(1.0, E, Z)
    py0, py1 = exact_solution(X, 0.0, Z), exact_solution(X, 1.0, Z)
    pz0, pz1 = exact_solution(X, E, 0.0), exact_solution(X, E, 1.0)
    Pxi = xi * px1 + (1.0 - xi) * px0
    Peta = eta * py1 + (1.0 - eta) * py0
    Pzeta = zeta * pz1 + (1.0 - zeta) * pz0
    u = (Pxi + Peta + Pzeta - Pxi * Peta - Pxi * Pzeta - Peta * Pzeta + Pxi * Peta * Pzeta)
    u = np.array(np.broadcast_to(u, (nz, ny, nx, 5)), dtype=np.float64, copy=True)
    ex = exact_grid(nx, ny, nz)
    for sl in ((slice(None), slice(None), 0), (slice(None), slice(None), nx - 1),
               (slice(None), 0), (slice(None), ny - 1), (0,), (nz - 1,)):
        u[sl] = ex[sl]
    return u


# NPB BT verification (verify.f, class S: 12^3, dt = 0.01, 60 iterations):
# the problem definition of the f4(ii) full-step check.
BT_STEPS = {"S": (12, 0.010, 60)}


def _dissipation(ue: np.ndarray, axis: int) -> np.ndarray:
    """NPB 5-case fourth-order dissipation of ``ue`` along ``axis`` (exact_rhs
    form), returned for indices 1..n-2 along that axis (others untouched = 0)."""
    n = ue.shape[axis]
    a = np.moveaxis(ue, axis, 0)
    out = np.zeros_like(a)
    out[1] = 5.0 * a[1] - 4.0 * a[2] + a[3]
    out[2] = -4.0 * a[1] + 6.0 * a[2] - 4.0 * a[3] + a[4]
    if n - 4 >= 3:
        out[3:n - 3] = (a[1:n - 5] - 4.0 * a[2:n - 4] + 6.0 * a[3:n - 3]
                        - 4.0 * a[4:n - 2] + a[5:n - 1])
    out[n - 3] = a[n - 5] - 4.0 * a[n - 4] + 6.0 * a[n - 3] - 4.0 * a[n - 2]
    out[n - 2] = a[n - 4] - 4.0 * a[n - 3] + 5.0 * a[n - 2]
    return np.moveaxis(out, 0, axis)


def exact_rhs(nx: int, ny: int, nz: int, dt: float = 0.0) -> np.ndarray:
    """NPB exact_rhs: forcing such that compute_rhs(exact_solution) ~ 0.

    Shape (nz, ny, nx, 5); zero on the boundary faces; ``dt`` is unused (the
    forcing does not depend on it) but accepted for symmetry.
    """
    if min(nx, ny, nz) < 6:
        raise ValueError("NAS dissipation needs n >= 6 in every dimension")
    c = GenConsts(nx, ny, nz, dt)
    ue = exact_grid(nx, ny, nz)                       # (nz, ny, nx, 5)
    forcing = np.zeros_like(ue)
    dtpp = 1.0 / ue[..., 0]
    buf = np.empty_like(ue)
    for m in range(1, 5):
        buf[..., m] = dtpp * ue[..., m]
    q = 0.5 * (buf[..., 1] * ue[..., 1] + buf[..., 2] * ue[..., 2] + buf[..., 3] * ue[..., 3])

    interior = (slice(1, nz - 1), slice(1, ny - 1), slice(1, nx - 1))

    # axis: 2 = xi (i), 1 = eta (j), 0 = zeta (k) in (k, j, i) array order.
    for axis, mom, t2, dt1, con in ((2, 1, c.tx2, c.dxt, "xx"),
                                   (1, 2, c.ty2, c.dyt, "yy"),
                                   (0, 3, c.tz2, c.dzt, "zz")):
        cuf = buf[..., mom] * buf[..., mom]
        b1 = buf[..., 1] * buf[..., 1] + buf[..., 2] * buf[..., 2] + buf[..., 3] * buf[..., 3]
        con1, con2, con3, con4, con5 = (getattr(c, con + f"con{n}") for n in range(1, 6))

        sp = list(interior)
        sp[axis] = slice(2, ue.shape[axis])
        sm = list(interior)
        sm[axis] = slice(0, ue.shape[axis] - 2)
        sp, sm = tuple(sp), tuple(sm)

        def P(a):  # value at +1 along axis, restricted to interior
            return a[sp]

        def M(a):  # value at -1 along axis, restricted to interior
            return a[sm]

        def C(a):
            return a[interior]

        def d2(a):
            return P(a) - 2.0 * C(a) + M(a)

        bmom = buf[..., mom]
        f = forcing[interior]
        for m in range(5):
            uem = ue[..., m]
            if m == 0:
                flux = -t2 * (P(ue[..., mom]) - M(ue[..., mom]))
                vis = 0.0
            elif m == mom:
                flux = -t2 * ((P(ue[..., mom]) * P(bmom) + c.c2 * (P(ue[..., 4]) - P(q)))
                              - (M(ue[..., mom]) * M(bmom) + c.c2 * (M(ue[..., 4]) - M(q))))
                vis = con1 * d2(bmom)
            elif m in (1, 2, 3):
                flux = -t2 * (P(uem) * P(bmom) - M(uem) * M(bmom))
                vis = con2 * d2(buf[..., m])
            else:
                flux = -t2 * (P(bmom) * (c.c1 * P(ue[..., 4]) - c.c2 * P(q))
                              - M(bmom) * (c.c1 * M(ue[..., 4]) - c.c2 * M(q)))
                vis = (0.5 * con3 * d2(b1) + con4 * d2(cuf) + con5 * d2(buf[..., 4]))
            f[..., m] = f[..., m] + flux + vis + dt1 * d2(uem)
        diss = _dissipation(ue, axis)[interior]
        f -= c.dssp * diss
        forcing[interior] = f

    forcing[interior] = -1.0 * forcing[interior]
    return forcing


@dataclass
class Inputs:
    bench: str
    cls: str
    nx: int
    ny: int
    nz: int
    dt: float
    seed: int
    u: np.ndarray        # (nz, ny, nx, 5)
    forcing: np.ndarray  # (nz, ny, nx, 5)


def make_inputs(nx: int, ny: int | None = None, nz: int | None = None, *,
                seed: int = 1, A: float = 1e-3, B: float = 0.0,
                dt: float = 0.001, bench: str = "", cls: str = "") -> Inputs:
    """u = exact * (1 + A*xi), forcing = exact_rhs + B*xi' (reading c11)."""
    ny = nx if ny is None else ny
    nz = nx if nz is None else nz
    ue = exact_grid(nx, ny, nz)
    u = ue if A == 0.0 else ue * (1.0 + A * uniform_pm1(seed, 0, ue.shape))
    f = exact_rhs(nx, ny, nz, dt)
    if B != 0.0:
        f = f + B * uniform_pm1(seed, 1, f.shape)
    return Inputs(bench, cls, nx, ny, nz, dt, seed,
                  np.ascontiguousarray(u), np.ascontiguousarray(f))


def make_class(bench: str, cls: str, *, seed: int = 1, A: float = 1e-3,
               B: float = 0.0) -> Inputs:
    n, dt = CLASSES[(bench, cls)]
    return make_inputs(n, n, n, seed=seed, A=A, B=B, dt=dt, bench=bench, cls=cls)


def config_name(bench: str, cls: str) -> str:
    n, _ = CLASSES[(bench, cls)]
    return f"{bench} compute_rhs class {cls} {n}^3 fp64"
