"""CPU oracle for the NAS BT/SP ``compute_rhs`` pass -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  It wraps the plain C
transcription in ``nas_oracle.c`` (NPB 3.x rhs.f as recalled in SURVEY.md
App. A; the paper names NPB BT/SP at PAPER.md L1330-1362, L1470-1488 but never
writes the loop nest) and shares no code with ``paper_conf_icpp_tiankexc16_b200``.

Arrays cross this wrapper in the *logical* layout ``(nz, ny, nx, 5)`` float64
(C order, component fastest), the layout ``nasgen`` produces; the wrapper pads
to the NAS-BT layout ``u[nz][ny'][nx'][5]`` the C code uses.

Pins: see ``tests/test_oracle_pins.py`` (P1-P6), ``test_oracle_exact_pins.py``
(P3), ``test_oracle_euler_pins.py`` (P7) and ``test_oracle_bt_pins.py`` (P8:
the full BT step reproduces NPB's class S/W/A verification norms, pinning the
NAS constants against NPB itself, reading c2).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "nas_oracle.c")
_SRCS = [_SRC, os.path.join(_HERE, "nas_bt.c")]
_HDR = os.path.join(_HERE, "nas_oracle.h")
_LIB = os.path.join(_HERE, "libnas_oracle.so")

# Strict IEEE: no FMA contraction, no reassociation (reading c6).
CFLAGS = ["-O2", "-std=c99", "-fPIC", "-shared", "-fopenmp",
          "-ffp-contract=off", "-fno-fast-math", "-fno-unsafe-math-optimizations"]

_FIELDS = (
    "dt c1 c2 c3 c4 c5 c1c2 c1c5 c3c4 conz1 con43 con16 dnxm1 dnym1 dnzm1 "
    "tx1 tx2 tx3 ty1 ty2 ty3 tz1 tz2 tz3 dx1 dx2 dx3 dx4 dx5 dy1 dy2 dy3 dy4 dy5 "
    "dz1 dz2 dz3 dz4 dz5 dssp dx1tx1 dx2tx1 dx3tx1 dx4tx1 dx5tx1 "
    "dy1ty1 dy2ty1 dy3ty1 dy4ty1 dy5ty1 dz1tz1 dz2tz1 dz3tz1 dz4tz1 dz5tz1 "
    "c3c4tx3 c3c4ty3 c3c4tz3 xxcon1 xxcon2 xxcon3 xxcon4 xxcon5 "
    "yycon1 yycon2 yycon3 yycon4 yycon5 zzcon1 zzcon2 zzcon3 zzcon4 zzcon5"
).split()


class OracleConsts(ctypes.Structure):
    _fields_ = [(f, ctypes.c_double) for f in _FIELDS]

    def as_dict(self) -> dict:
        return {f: getattr(self, f) for f in _FIELDS}


_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle shared library in-tree with gcc (idempotent)."""
    stale = (not os.path.exists(_LIB) or
             os.path.getmtime(_LIB) < max(os.path.getmtime(p) for p in _SRCS + [_HDR]))
    if force or stale:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, *_SRCS, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            lib.oracle_set_constants.argtypes = [ctypes.c_int] * 3 + [
                ctypes.c_double, ctypes.POINTER(OracleConsts)]
            lib.oracle_set_constants.restype = ctypes.c_int
            lib.oracle_padded.argtypes = [ctypes.c_int]
            lib.oracle_padded.restype = ctypes.c_int
            dp = ctypes.POINTER(ctypes.c_double)
            lib.oracle_compute_rhs.argtypes = [ctypes.c_int] * 3 + [
                ctypes.POINTER(OracleConsts), dp, dp, dp, ctypes.c_int]
            lib.oracle_compute_rhs.restype = ctypes.c_int
            lib.oracle_compute_aux.argtypes = [ctypes.c_int] * 3 + [
                ctypes.POINTER(OracleConsts), dp, dp, ctypes.c_int]
            lib.oracle_compute_aux.restype = ctypes.c_int
            lib.oracle_rhs_sumsq.argtypes = [ctypes.c_int] * 3 + [dp, dp]
            lib.oracle_rhs_sumsq.restype = ctypes.c_int
            lib.oracle_seismic_dz.argtypes = [ctypes.c_int] * 3 + [dp] * 4 + [ctypes.c_double]
            lib.oracle_seismic_dz.restype = ctypes.c_int
            cp = ctypes.POINTER(OracleConsts)
            lib.oracle_bt_solve.argtypes = [ctypes.c_int] * 4 + [cp, dp, dp, dp]
            lib.oracle_bt_solve.restype = ctypes.c_int
            lib.oracle_bt_add.argtypes = [ctypes.c_int] * 3 + [dp, dp]
            lib.oracle_bt_add.restype = ctypes.c_int
            lib.oracle_bt_run.argtypes = [ctypes.c_int] * 3 + [cp, dp, dp, dp, dp, ctypes.c_int,
                                                                ctypes.c_int]
            lib.oracle_bt_run.restype = ctypes.c_int
            lib.oracle_error_norm.argtypes = [ctypes.c_int] * 3 + [dp, dp, dp]
            lib.oracle_error_norm.restype = ctypes.c_int
            _lib = lib
    return _lib


def set_constants(nx: int, ny: int, nz: int, dt: float) -> OracleConsts:
    """NPB set_constants as computed by the C oracle."""
    c = OracleConsts()
    if _load().oracle_set_constants(nx, ny, nz, dt, ctypes.byref(c)) != 0:
        raise ValueError("oracle_set_constants: bad extents")
    return c


def padded(n: int) -> int:
    return _load().oracle_padded(n)


def to_nas(a: np.ndarray) -> np.ndarray:
    """(nz, ny, nx, 5) -> zero-padded NAS-BT layout (nz, ny', nx', 5)."""
    nz, ny, nx, _ = a.shape
    out = np.zeros((nz, padded(ny), padded(nx), 5), dtype=np.float64)
    out[:, :ny, :nx, :] = a
    return out


def from_nas(a: np.ndarray, nx: int, ny: int) -> np.ndarray:
    return np.ascontiguousarray(a[:, :ny, :nx, :])


def compute_rhs(u: np.ndarray, forcing: np.ndarray, dt: float | None = None,
                consts: OracleConsts | None = None, threads: int = 1) -> np.ndarray:
    """One NAS compute_rhs pass on the CPU.

    ``u`` and ``forcing`` have logical shape (nz, ny, nx, 5) float64.  Either
    ``dt`` (constants from NAS set_constants) or an explicit ``consts`` must be
    given.  Returns rhs with the same logical shape.
    """
    if u.shape != forcing.shape or u.ndim != 4 or u.shape[3] != 5:
        raise ValueError("u / forcing must both have shape (nz, ny, nx, 5)")
    nz, ny, nx, _ = u.shape
    if consts is None:
        if dt is None:
            raise ValueError("give dt or consts")
        consts = set_constants(nx, ny, nz, dt)
    un = to_nas(np.asarray(u, dtype=np.float64))
    fn = to_nas(np.asarray(forcing, dtype=np.float64))
    rn = np.zeros_like(un)
    dp = ctypes.POINTER(ctypes.c_double)
    rc = _load().oracle_compute_rhs(nx, ny, nz, ctypes.byref(consts),
                                    un.ctypes.data_as(dp), fn.ctypes.data_as(dp),
                                    rn.ctypes.data_as(dp), int(threads))
    if rc != 0:
        raise ValueError(f"oracle_compute_rhs failed ({rc}): extents must be >= 6")
    return from_nas(rn, nx, ny)


def compute_aux(u: np.ndarray, naux: int = 6, dt: float | None = None,
                consts: OracleConsts | None = None) -> np.ndarray:
    """NAS compute_rhs step 0 fields at every point.

    Returns shape (nz, ny, nx, naux): rho_i, us, vs, ws, square, qs (BT rhs.f
    order) and, for naux = 7, SP's speed = sqrt(c1c2*rho_i*(u5 - square)).
    ``dt`` only selects the constants (c1c2); it does not enter step 0."""
    nz, ny, nx, _ = u.shape
    if consts is None:
        consts = set_constants(nx, ny, nz, 1.0 if dt is None else dt)
    un = to_nas(np.asarray(u, dtype=np.float64))
    an = np.zeros(un.shape[:3] + (naux,), dtype=np.float64)
    dp = ctypes.POINTER(ctypes.c_double)
    rc = _load().oracle_compute_aux(nx, ny, nz, ctypes.byref(consts), un.ctypes.data_as(dp),
                                    an.ctypes.data_as(dp), int(naux))
    if rc != 0:
        raise ValueError("oracle_compute_aux: bad arguments (naux must be 6 or 7)")
    return np.ascontiguousarray(an[:, :ny, :nx, :])


def rhs_sumsq(rhs: np.ndarray) -> np.ndarray:
    """NPB error.f rhs_norm numerator: per component, the sum of rhs^2 over
    the interior points, in the Fortran loop order."""
    nz, ny, nx, _ = rhs.shape
    rn = to_nas(np.asarray(rhs, dtype=np.float64))
    out = np.zeros(5, dtype=np.float64)
    dp = ctypes.POINTER(ctypes.c_double)
    if _load().oracle_rhs_sumsq(nx, ny, nz, rn.ctypes.data_as(dp), out.ctypes.data_as(dp)) != 0:
        raise ValueError("oracle_rhs_sumsq: extents must be >= 3")
    return out


def seismic_dz(vz1: np.ndarray, vz2: np.ndarray, vz3: np.ndarray, h: float,
               init: np.ndarray | None = None) -> np.ndarray:
    """PAPER.md Fig. 8 dz loop.  Arrays are indexed
    [k, j, i] (C order of Fortran vz(i,j,k)); points outside the loop ranges
    keep ``init`` (default NaN)."""
    nz, ny, nx = vz1.shape
    out = (np.full((nz, ny, nx), np.nan) if init is None
           else np.array(init, dtype=np.float64, copy=True))
    a = [np.ascontiguousarray(v, dtype=np.float64) for v in (vz1, vz2, vz3)]
    dp = ctypes.POINTER(ctypes.c_double)
    if _load().oracle_seismic_dz(nx, ny, nz, *(v.ctypes.data_as(dp) for v in a),
                                 out.ctypes.data_as(dp), float(h)) != 0:
        raise ValueError("oracle_seismic_dz: extents must be >= 2")
    return out


# ---- the full NPB BT time step (nas_bt.c) -------------

def _nas_scratch(nz: int, ny: int, nx: int, ncomp: int) -> np.ndarray:
    return np.zeros((nz, padded(ny), padded(nx), ncomp), dtype=np.float64)


def bt_solve(direction: int, u: np.ndarray, rhs: np.ndarray, dt: float) -> np.ndarray:
    """NPB BT x_solve (0), y_solve (1) or z_solve (2) applied to ``rhs``
    (logical (nz, ny, nx, 5)); the aux fields come from compute_aux(u)."""
    nz, ny, nx, _ = u.shape
    consts = set_constants(nx, ny, nz, dt)
    un = to_nas(np.asarray(u, dtype=np.float64))
    rn = to_nas(np.asarray(rhs, dtype=np.float64))
    an = _nas_scratch(nz, ny, nx, 6)
    dp = ctypes.POINTER(ctypes.c_double)
    L = _load()
    if L.oracle_compute_aux(nx, ny, nz, ctypes.byref(consts), un.ctypes.data_as(dp),
                            an.ctypes.data_as(dp), 6) != 0:
        raise ValueError("oracle_compute_aux failed")
    if L.oracle_bt_solve(int(direction), nx, ny, nz, ctypes.byref(consts), un.ctypes.data_as(dp),
                         an.ctypes.data_as(dp), rn.ctypes.data_as(dp)) != 0:
        raise ValueError("oracle_bt_solve failed")
    return from_nas(rn, nx, ny)


def bt_run(u0: np.ndarray, forcing: np.ndarray, dt: float, niter: int,
           threads: int = 1) -> tuple[np.ndarray, np.ndarray]:
    """``niter`` NPB BT adi steps from ``u0``; returns (u, rhs of the last
    step after the solves), logical layout."""
    nz, ny, nx, _ = u0.shape
    consts = set_constants(nx, ny, nz, dt)
    un = to_nas(np.asarray(u0, dtype=np.float64))
    fn = to_nas(np.asarray(forcing, dtype=np.float64))
    rn = np.zeros_like(un)
    an = _nas_scratch(nz, ny, nx, 6)
    dp = ctypes.POINTER(ctypes.c_double)
    if _load().oracle_bt_run(nx, ny, nz, ctypes.byref(consts), un.ctypes.data_as(dp),
                             fn.ctypes.data_as(dp), rn.ctypes.data_as(dp), an.ctypes.data_as(dp),
                             int(niter), int(threads)) != 0:
        raise ValueError("oracle_bt_run failed")
    return from_nas(un, nx, ny), from_nas(rn, nx, ny)


def error_norm(u: np.ndarray, u_exact: np.ndarray) -> np.ndarray:
    """NPB error_norm: per component sqrt(sum_all (u - u_exact)^2 / prod(n-2))."""
    nz, ny, nx, _ = u.shape
    un = to_nas(np.asarray(u, dtype=np.float64))
    en = to_nas(np.asarray(u_exact, dtype=np.float64))
    out = np.zeros(5, dtype=np.float64)
    dp = ctypes.POINTER(ctypes.c_double)
    if _load().oracle_error_norm(nx, ny, nz, un.ctypes.data_as(dp), en.ctypes.data_as(dp),
                                 out.ctypes.data_as(dp)) != 0:
        raise ValueError("oracle_error_norm failed")
    return out


def bt_verify_norms(u0: np.ndarray, forcing: np.ndarray, u_exact: np.ndarray, dt: float,
                    niter: int, threads: int = 1) -> tuple[np.ndarray, np.ndarray]:
    """NPB BT verify: after ``niter`` steps, xce = error_norm(u) and
    xcr = rhs_norm(compute_rhs(u)) / dt."""
    nz, ny, nx, _ = u0.shape
    u, _ = bt_run(u0, forcing, dt, niter, threads)
    xce = error_norm(u, u_exact)
    r = compute_rhs(u, forcing, dt=dt, threads=threads)
    xcr = np.sqrt(rhs_sumsq(r) / ((nx - 2) * (ny - 2) * (nz - 2))) / dt
    return xce, xcr
