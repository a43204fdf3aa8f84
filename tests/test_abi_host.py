"""Host-side checks of the C ABI that need no GPU: the library builds for
sm_100a, loads, exports every symbol include/safara.h declares, and its host
logic (descriptor validation = the dim/small clause check, PAPER.md
L1275-1291; NPB coefficients; canonical pitch) behaves as documented."""
import ctypes
import subprocess

import pytest

import paper_conf_icpp_tiankexc16_b200 as sr
from paper_conf_icpp_tiankexc16_b200 import _abi, build


@pytest.fixture(scope="module")
def L():
    build.build()
    return _abi.lib()


def test_exports_every_header_symbol(L):
    syms = _abi.header_symbols()
    assert len(syms) >= 12
    for s in syms:
        assert hasattr(L, s), s
    out = subprocess.run(["nm", "-D", "--defined-only", _abi.LIB_PATH], capture_output=True,
                         text=True).stdout
    for s in syms:
        assert f" T {s}" in out, s


def test_sass_is_sm100a_with_tma():
    build.build()
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", _abi.LIB_PATH],
                          capture_output=True, text=True).stdout
    assert "sm_100a" in sass
    assert "UTMALDG" in sass          # cp.async.bulk.tensor (TMA) loads
    assert "DFMA" in sass and "DMUL" in sass
    assert "HMMA" not in sass         # no legacy tensor-core path


def test_ptxas_zero_spills():
    """ptxas -v of the current build: the production kernels (the round-2
    warp-specialised NAS instance the bench runs, its aux variant, and the
    round-1 production kernel) have no stack frame and no spill bytes."""
    from paper_conf_icpp_tiankexc16_b200 import safara_tune as st
    build.build()
    path = build.os.path.join(build.BUILD, "ptxas.txt")
    if not build.os.path.exists(path):
        build.build(force=True)
    info = st.ptxas_info(open(path).read())
    for name in ("rhs_kernel_fast_ws_ud", "rhs_kernel_fast_ws_ud_aux", "rhs_kernel_fast_ud",
                 "rhs_kernel_fast_ud_aux"):
        key = f"_ZN6safara{len(name)}{name}E14CUtensorMap_stS0_NS_6ParamsE"
        assert key in info, name
        k = info[key]
        assert k["spill_st"] == 0 and k["spill_ld"] == 0 and k["stack"] == 0, (name, k)


def test_pitch_and_canonical_dims(L):
    for nx, p in ((12, 16), (36, 40), (64, 64), (102, 104), (162, 168)):
        assert sr.pitch(nx) == p
        d = sr.canonical_dims(nx, nx, nx)
        assert (d.sy, d.sm, d.sk) == (p, nx * p, 5 * nx * p)
        assert sr.validate_dims(d, nx) == 0


def test_validation_errors(L):
    d = sr.canonical_dims(12, 12, 12)
    assert sr.validate_dims(d, 12) == 0
    bad = _abi.Dims(5, 12, 12, d.sy, d.sm, d.sk)
    assert sr.validate_dims(bad, 12) == -2                     # SHAPE: n < 6
    bad = _abi.Dims(12, 12, 12, 10, d.sm, d.sk)
    assert sr.validate_dims(bad, 12) == -3                     # LAYOUT: sy < nx
    bad = _abi.Dims(12, 12, 12, 16, 100, d.sk)
    assert sr.validate_dims(bad, 12) == -3                     # LAYOUT: m overlaps j
    bad = _abi.Dims(12, 12, 12, 13, 13 * 12, 13 * 60)
    assert sr.validate_dims(bad, 12) == -4                     # ALIGN: odd stride
    big = sr.canonical_dims(1000, 1000, 20)
    assert sr.validate_dims(big, 20) == 0
    assert sr.validate_dims(big, 500) == -5                    # TOO_LARGE: small is false
    # SP-native [m][k][j][i]: k stride below m stride is a valid descriptor.
    nx = ny = nz = 12
    sp = _abi.Dims(nx, ny, nz, 16, 16 * ny * nz, 16 * ny)
    assert sr.validate_dims(sp, nz) == 0


def test_canonical_too_large(L):
    d = _abi.Dims()
    assert L.safara_dims_canonical(2000, 2000, 200, ctypes.byref(d)) == -5


def test_strerror(L):
    for code in range(0, -9, -1):
        assert len(_abi.strerror(code)) > 5
    assert "unknown" in _abi.strerror(-99)


def test_coeffs_match_nas_constants(L):
    """The library's own set_constants equals the oracle's, value for value
    (both follow SURVEY App. B; they share no code)."""
    import oracle
    for n, dt in ((12, 0.01), (36, 0.0015), (162, 0.0001)):
        c = sr.coeffs_nas(n, n + 2, n + 4, dt)
        o = oracle.set_constants(n, n + 2, n + 4, dt)
        assert c.dt == o.dt and c.dssp == o.dssp and c.c1 == o.c1 and c.c2 == o.c2
        assert c.con43 == o.con43
        assert (c.tx2, c.ty2, c.tz2) == (o.tx2, o.ty2, o.tz2)
        for m in range(5):
            assert c.dxt[m] == getattr(o, f"dx{m + 1}tx1")
            assert c.dyt[m] == getattr(o, f"dy{m + 1}ty1")
            assert c.dzt[m] == getattr(o, f"dz{m + 1}tz1")
            for ax in ("xx", "yy", "zz"):
                assert getattr(c, ax + "con")[m] == getattr(o, f"{ax}con{m + 1}")


def test_compute_without_init_fails_loudly(L):
    # No GPU here: the compute entry must return an error, never run on the CPU.
    rc = L.safara_rhs(1 << 20, 2 << 20, 3 << 20, 12, 12, 12, ctypes.byref(_abi.Coeffs()), None)
    assert rc < 0


def test_peer_struct_layout_matches_header(tmp_path):
    """safara_peer_t as the C compiler lays it out == the ctypes mirror."""
    src = tmp_path / "peer.c"
    src.write_text('#include <stddef.h>\n#include <stdio.h>\n#include "safara.h"\n'
                   'int main(void){printf("%zu %zu %zu %zu %zu %zu %zu %zu %zu\\n",'
                   'sizeof(safara_peer_t), offsetof(safara_peer_t,u_lo),'
                   'offsetof(safara_peer_t,u_hi), offsetof(safara_peer_t,k0_lo),'
                   'offsetof(safara_peer_t,k0_hi), offsetof(safara_peer_t,flags),'
                   'offsetof(safara_peer_t,flags_lo), offsetof(safara_peer_t,flags_hi),'
                   'offsetof(safara_peer_t,epoch));return 0;}\n')
    exe = tmp_path / "peer"
    inc = build.INCLUDE
    subprocess.run(["gcc", "-I", inc, str(src), "-o", str(exe)], check=True)
    got = [int(x) for x in subprocess.run([str(exe)], capture_output=True,
                                          text=True).stdout.split()]
    P = _abi.Peer
    want = [ctypes.sizeof(P)] + [getattr(P, f).offset for f in
                                  ("u_lo", "u_hi", "k0_lo", "k0_hi", "flags", "flags_lo",
                                   "flags_hi", "epoch")]
    assert got == want


def test_peer_neighbours_and_struct():
    from paper_conf_icpp_tiankexc16_b200 import dist as sd
    nb = [sd.neighbours(162, 8, r) for r in range(8)]
    assert nb[0]["lo"] is None and nb[0]["k0_hi"] == 21 and nb[7]["hi"] is None
    for r in range(1, 8):
        # the lower neighbour's slab ends where this one starts, and owns >= 2 planes
        assert nb[r]["k0_lo"] == nb[r - 1]["k0"]
        assert nb[r]["k0"] - nb[r]["k0_lo"] >= 2
        assert nb[r - 1]["k0_hi"] == nb[r]["k0"]
    pr = sd.peer_struct(nb[3], 0x1000, 0x2000, 0x3000, 0x4000, 0x5000, 0)
    assert pr.u_lo == 0x1000 and pr.u_hi == 0x2000 and pr.flags_lo is None  # epoch 0: no flags
    pr = sd.peer_struct(nb[0], None, 0x2000, 0x3000, None, 0x5000, 7)
    assert pr.u_lo is None and pr.flags_hi == 0x5000 and pr.epoch == 7 and pr.k0_hi == 21


def test_rhs_peer_rejects_bad_arguments_without_gpu(L):
    """Argument checks run before any device work (no GPU needed)."""
    d = sr.canonical_dims(12, 12, 12)
    c = sr.coeffs_nas(12, 12, 12, 0.01)
    pr = _abi.Peer()
    # NULL peer struct / NULL dims
    assert L.safara_rhs_peer(16, 16, 16, None, 0, 6, ctypes.byref(pr), ctypes.byref(c), 0,
                             None) != 0
    assert L.safara_rhs_peer(16, 16, 16, ctypes.byref(d), 0, 6, None, ctypes.byref(c), 0,
                             None) != 0
