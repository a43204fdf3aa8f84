"""Pins for the oracle's 355.seismic dz loop (Fig. 8;
SURVEY §8(f) f4(i)), none retyping its expression:

S1  fields linear in k (vz_n = a_n k + g_n(i,j), dyadic a_n and h) give
    value_dz = a_1/h + a_2/h + a_3/h exactly at every written point -- pins the
    k-1 neighbour, the division and the k-independence.
S2  one array at a time: only vz_n varying in k gives a_n/h -- no array is
    dropped, doubled or swapped.
S3  loop ranges (zero lower bounds): j = 0, i = nx-1 and k = 0 are never
    written; everything else is.
S4  exact-rational brute force on a tiny dyadic grid: the fp64 result is
    within 3 ulp-scale roundings of the exact value.
"""
from fractions import Fraction

import numpy as np

import oracle


def _grid(nx, ny, nz):
    return np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")


def test_s1_linear_in_k_exact():
    nx, ny, nz, h = 7, 5, 9, 0.25
    k, j, i = _grid(nx, ny, nz)
    a = (0.5, -1.5, 2.0)
    v = [a[n] * k + (i * 3 + j * 7 + n) * 0.125 for n in range(3)]
    out = oracle.seismic_dz(*v, h)
    expect = a[0] / h + a[1] / h + a[2] / h
    w = out[1:, 1:, :-1]
    assert np.array_equal(w, np.full_like(w, expect))


def test_s2_each_array_contributes_once():
    nx, ny, nz, h = 6, 4, 5, 0.5
    k, j, i = _grid(nx, ny, nz)
    for n, a in ((0, 1.0), (1, 2.0), (2, 4.0)):
        v = [np.full((nz, ny, nx), 3.0) + 0.25 * (i + j) for _ in range(3)]
        v[n] = v[n] + a * k
        out = oracle.seismic_dz(*v, h)
        assert np.array_equal(out[1:, 1:, :-1], np.full((nz - 1, ny - 1, nx - 1), a / h))


def test_s3_loop_ranges():
    nx, ny, nz = 6, 5, 4
    r = np.random.default_rng(1)
    v = [r.random((nz, ny, nx)) for _ in range(3)]
    out = oracle.seismic_dz(*v, 0.1)
    written = ~np.isnan(out)
    assert not written[0].any() and not written[:, 0].any() and not written[:, :, nx - 1].any()
    assert written[1:, 1:, :nx - 1].all()


def test_s4_exact_rational_brute_force():
    nx, ny, nz, h = 4, 3, 4, 0.375
    r = np.random.default_rng(2)
    v = [np.round(r.random((nz, ny, nx)) * 1024) / 1024 for _ in range(3)]
    out = oracle.seismic_dz(*v, h)
    H = Fraction(h)
    for kk in range(1, nz):
        for jj in range(1, ny):
            for ii in range(nx - 1):
                ex = sum((Fraction(v[n][kk, jj, ii]) - Fraction(v[n][kk - 1, jj, ii])) / H
                         for n in range(3))
                got = out[kk, jj, ii]
                assert abs(Fraction(got) - ex) <= Fraction(4 * 2.0 ** -52) * (abs(ex) + 4)
