"""Pins of the oracle's spatial operators (O1) — CPU only.

The paper fixes only the stencil size: "operators with a 3D stencil width of 8",
"25 data read accesses" (§5), a "25-point stencil" (§3.1).
These tests pin the oracle's coefficient table and operators to that definition
without re-typing the oracle:
* the table equals the fp32 rounding of the exact rationals that
  tests/golden/make_coefficients.py derives from the Taylor systems;
* Lambda and D+/- are exact on polynomials of the degrees an 8th-order operator
  must differentiate exactly (up to the fp32 rounding of the coefficients).
"""
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "stencil_coefficients.txt")


def _golden():
    vals = {}
    for line in open(GOLD):
        if line.startswith("#") or not line.strip():
            continue
        k, num, den = line.split()
        vals[k] = Fraction(int(num), int(den))
    return vals


def test_coefficients_are_fp32_of_exact_rationals():
    c, d = oracle.coef()
    g = _golden()
    for m in range(5):
        assert c[m] == float(np.float32(float(g[f"c{m}"]))), m
    for m in range(4):
        assert d[m] == float(np.float32(float(g[f"d{m + 1}"]))), m


def test_coefficients_satisfy_taylor_moments():
    c, d = oracle.coef()
    # centred: row sum 0, second moment 1 (per axis), higher even moments 0 -- to fp32 rounding
    assert abs(c[0] + 2 * sum(c[1:])) < 1e-6
    assert abs(sum(c[m] * m ** 2 for m in range(1, 5)) - 1.0) < 1e-6
    for k in (2, 3, 4):
        assert abs(sum(c[m] * m ** (2 * k) for m in range(1, 5))) < 1e-6 * 4 ** (2 * k)
    # staggered: first moment 1, odd higher moments 0
    assert abs(sum(d[m - 1] * (2 * m - 1) for m in range(1, 5)) - 1.0) < 1e-6
    for k in (1, 2, 3):
        assert abs(sum(d[m - 1] * (2 * m - 1) ** (2 * k + 1) for m in range(1, 5))) < 1e-6 * 7 ** (2 * k + 1)


def _poly(deg, rng, n):
    return rng.standard_normal(deg + 1) / np.arange(1, deg + 2)


@pytest.mark.parametrize("axis", [0, 1, 2])
def test_laplacian_exact_on_degree9_polynomials(axis):
    """Lambda u / h^2 reproduces u'' for polynomials of degree <= 9 along each axis
    (interior points, 4 away from the zero ghosts)."""
    n = 24
    g = oracle.Grid(n, n, n, h=1.0, dt=1.0)
    rng = np.random.default_rng(1)
    coefs = _poly(9, rng, n)
    s = (np.arange(n) - n / 2) / 8.0  # normalised coordinate, |s| <= 1.5
    p = np.polynomial.Polynomial(coefs)
    prof = p(s)
    d2 = p.deriv(2)(s) / 64.0  # d^2/di^2 = (1/8^2) d^2/ds^2
    shape = [1, 1, 1]
    shape[2 - axis] = n
    u = np.broadcast_to(prof.reshape(shape), (n, n, n)).copy()
    out = oracle.lap(g, u)
    sl = [slice(4, n - 4)] * 3
    ref = np.broadcast_to(d2.reshape(shape), (n, n, n))[tuple(sl)]
    err = np.abs(out[tuple(sl)] - ref).max()
    scale = np.abs(u).max() * 8.0  # sum |c_m| * max|u|
    assert err < 2e-6 * scale, err


def test_laplacian_sums_three_axes_and_zero_ghosts():
    n = 16
    g = oracle.Grid(n, n, n, h=1.0, dt=1.0)
    c, _ = oracle.coef()
    u = np.zeros((n, n, n))
    u[0, 0, 0] = 1.0  # corner spike: half the stencil falls on zero ghosts
    out = oracle.lap(g, u)
    assert out[0, 0, 0] == pytest.approx(3 * c[0])
    for m in range(1, 5):
        assert out[0, 0, m] == pytest.approx(c[m])
        assert out[0, m, 0] == pytest.approx(c[m])
        assert out[m, 0, 0] == pytest.approx(c[m])
    assert out[1, 1, 0] == 0.0
    assert np.count_nonzero(out) == 1 + 3 * 4


@pytest.mark.parametrize("axis", [0, 1, 2])
@pytest.mark.parametrize("plus", [True, False])
def test_staggered_derivative_exact_on_degree8_polynomials(axis, plus):
    """h D+ f at i+1/2 and h D- g at i reproduce the first derivative of polynomials of
    degree <= 8 at the staggered positions (integer index i of a half-node field holds i+1/2)."""
    n = 24
    g = oracle.Grid(n, n, n, h=1.0, dt=1.0)
    rng = np.random.default_rng(2)
    p = np.polynomial.Polynomial(_poly(8, rng, n))
    i = np.arange(n, dtype=np.float64)
    pos_in = i if plus else i + 0.5   # D+ reads an integer-node field, D- a half-node field
    pos_out = i + 0.5 if plus else i
    f_in = p((pos_in - n / 2) / 8.0)
    ref = p.deriv(1)((pos_out - n / 2) / 8.0) / 8.0
    shape = [1, 1, 1]
    shape[2 - axis] = n
    f = np.broadcast_to(f_in.reshape(shape), (n, n, n)).copy()
    out = oracle.dstag(g, axis, plus, f)
    sl = [slice(4, n - 4)] * 3
    refb = np.broadcast_to(ref.reshape(shape), (n, n, n))[tuple(sl)]
    err = np.abs(out[tuple(sl)] - refb).max()
    assert err < 2e-6 * np.abs(f).max() * 2.5, err


def test_staggered_operators_are_negative_adjoints():
    """sum f (D- q) = - sum q (D+ f) with zero ghosts (summation by parts, O8 energy)."""
    n = 12
    g = oracle.Grid(n, n, n, h=1.0, dt=1.0)
    rng = np.random.default_rng(3)
    f = rng.standard_normal((n, n, n))
    q = rng.standard_normal((n, n, n))
    for ax in range(3):
        lhs = np.sum(f * oracle.dstag(g, ax, False, q))
        rhs = -np.sum(q * oracle.dstag(g, ax, True, f))
        assert lhs == pytest.approx(rhs, rel=1e-12, abs=1e-12)
