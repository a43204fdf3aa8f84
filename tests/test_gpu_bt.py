"""GPU: a whole NPB BT time step through the C ABI (SURVEY §8(f) f4(ii):
safara_bt_step = safara_rhs_aux + safara_bt_solve x/y/z + safara_bt_add,
safara_error_norm, safara_rhs_rms) against the oracle's BT step
(oracle/nas_bt.c) and NPB's own verification values
(tests/golden/npb_bt_verify.txt, NPB epsilon 1e-8)."""
import numpy as np
import pytest
import torch

import nasgen
import oracle
import paper_conf_icpp_tiankexc16_b200 as sr
from test_oracle_bt_pins import EPSILON, golden

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _init():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sr.init(0)


def _state(n, dt, u0=None):
    u0 = nasgen.nas_initialize(n, n, n) if u0 is None else u0
    f = nasgen.exact_rhs(n, n, n, dt)
    return sr.BtState(sr.pack(u0), sr.pack(f), n, dt), u0, f


@pytest.mark.parametrize("direction", [0, 1, 2])
def test_line_solve_bitwise_vs_oracle(direction):
    """Each direction's block-tridiagonal line solve is bit-identical to the
    oracle's on the same u and rhs (aux from the STRICT pass)."""
    n, dt = 13, 0.01
    inp = nasgen.make_inputs(n, 11, 9, seed=4, A=1e-3, B=1e-2, dt=dt)
    nz, ny, nx, _ = inp.u.shape
    st = sr.BtState(sr.pack(inp.u), sr.pack(inp.forcing), nx, dt)
    sr.rhs_aux(st.u, st.forcing, st.rhs, st.aux, nx, st.coeffs, strict=True)
    st.solve(direction)
    torch.cuda.synchronize()
    r = oracle.compute_rhs(inp.u, inp.forcing, dt=dt)
    want = oracle.bt_solve(direction, inp.u, r, dt)
    assert np.array_equal(sr.unpack(st.rhs, nx), want)


def test_bt_class_s_strict_bitwise_trajectory():
    """60 STRICT steps of class S: u after every 20 steps is bit-identical to
    the oracle's run (compute_rhs, aux, solves and add all bitwise)."""
    g = golden()["S"]
    n, dt = g["n"], g["dt"]
    st, u0, f = _state(n, dt)
    u = u0
    for block in range(3):
        for _ in range(20):
            st.step(strict=True)
        torch.cuda.synchronize()
        u, _ = oracle.bt_run(u, f, dt, 20)
        assert np.array_equal(sr.unpack(st.u, n), u), f"diverged in steps {20 * block}..{20 * block + 19}"


@pytest.mark.parametrize("cls,strict", [("S", True), ("S", False), ("W", False), ("A", False)])
def test_bt_npb_verification(cls, strict):
    """NPB BT verify on the GPU: error and rhs norms within NPB's 1e-8."""
    g = golden()[cls]
    n, dt, niter = g["n"], g["dt"], g["niter"]
    st, _, _ = _state(n, dt)
    l0 = sr.launch_count()
    for _ in range(niter):
        st.step(strict=strict)
    assert sr.launch_count() - l0 == 5 * niter
    ue = sr.pack(nasgen.exact_grid(n, n, n))
    xce, xcr = st.verify_norms(ue, strict=strict)
    torch.cuda.synchronize()
    xce, xcr = xce.cpu().numpy(), xcr.cpu().numpy()
    rel_e = np.abs(xce - g["xce"]) / g["xce"]
    rel_r = np.abs(xcr - g["xcr"]) / g["xcr"]
    assert (rel_e <= EPSILON).all(), rel_e
    assert (rel_r <= EPSILON).all(), rel_r


def test_bt_argument_checks():
    import ctypes
    from paper_conf_icpp_tiankexc16_b200 import _abi
    st, _, _ = _state(12, 0.01)
    L = _abi.lib()
    assert L.safara_bt_solve(3, st.u.data_ptr(), st.aux.data_ptr(), st.rhs.data_ptr(),
                             st.work.data_ptr(), ctypes.byref(st.dims), ctypes.byref(st.bt),
                             None) == -1
    # rhs aliasing u
    assert L.safara_bt_solve(0, st.u.data_ptr(), st.aux.data_ptr(), st.u.data_ptr(),
                             st.work.data_ptr(), ctypes.byref(st.dims), ctypes.byref(st.bt),
                             None) == -1
    assert L.safara_bt_work_doubles(5, 12, 12) == -2
