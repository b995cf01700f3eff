"""Pins of the source wavelet (O10, O11) -- CPU only.

The paper never names the wavelet ("f is the point source"); BASELINE.json names the
Ricker wavelet.  inputs.ricker / inputs.ricker_integral / inputs.source_series produce the
samples BOTH sides inject, so they are pinned here against properties of the Ricker wavelet
that do not restate its formula:

* shape: w(t0) = 1 (peak), zeros at t0 +- 1/(sqrt(2) pi fp), minima -2 exp(-3/2) at
  t0 +- sqrt(3/2)/(pi fp), even about t0;
* peak frequency: the amplitude spectrum |W(f)| of a Ricker wavelet peaks at fp
  (located here with numpy's FFT, a library routine);
* antiderivative: ricker_integral(t) - ricker_integral(t_a) equals the quadrature of
  ricker over [t_a, t] (scipy.integrate.quad), and ricker_integral -> 0 on both tails;
* the injected series s[n] (O11): ISO samples w at n dt, ACOUSTIC / ELASTIC the integral
  at (n + 1/2) dt, both with dt rounded to fp32 as the library receives it.
"""
import math

import numpy as np
import pytest
from scipy.integrate import quad

from paper_conf_ppopp_qawasmehchc15_b200 import inputs

FP = [10.0, 15.0, 25.0]


@pytest.mark.parametrize("fp", FP)
def test_ricker_shape(fp):
    t0 = 1.5 / fp
    assert inputs.ricker(t0, fp) == pytest.approx(1.0, abs=1e-15)
    tz = 1.0 / (math.sqrt(2.0) * math.pi * fp)
    for s in (-1, 1):
        assert abs(float(inputs.ricker(t0 + s * tz, fp))) < 1e-14
        tm = t0 + s * math.sqrt(1.5) / (math.pi * fp)
        assert float(inputs.ricker(tm, fp)) == pytest.approx(-2.0 * math.exp(-1.5), rel=1e-13)
        # tm is a minimum: values on both sides are larger
        eps = 1e-4 / fp
        assert inputs.ricker(tm - eps, fp) > inputs.ricker(tm, fp) < inputs.ricker(tm + eps, fp)
    t = np.linspace(0.0, t0, 257)
    assert np.allclose(inputs.ricker(t0 - t, fp), inputs.ricker(t0 + t, fp), rtol=0, atol=1e-12)
    # default delay t0 = 1.5 / fp makes the start negligible (|w(0)| ~ 1e-8, O10)
    assert abs(float(inputs.ricker(0.0, fp))) < 1e-7


@pytest.mark.parametrize("fp", FP)
def test_ricker_peak_frequency(fp):
    dt, n = 1e-4, 1 << 18  # 0.038 Hz resolution
    w = inputs.ricker(np.arange(n) * dt, fp)
    spec = np.abs(np.fft.rfft(w))
    freqs = np.fft.rfftfreq(n, dt)
    assert freqs[np.argmax(spec)] == pytest.approx(fp, abs=0.05)


@pytest.mark.parametrize("fp", FP)
def test_ricker_integral_is_the_antiderivative(fp):
    t0 = 1.5 / fp
    ta = 0.0
    for t in np.linspace(0.0, 4.0 * t0, 23):
        val, _ = quad(lambda s: float(inputs.ricker(s, fp)), ta, float(t), epsabs=1e-14, epsrel=1e-12,
                      limit=200)
        got = float(inputs.ricker_integral(t, fp) - inputs.ricker_integral(ta, fp))
        assert got == pytest.approx(val, abs=1e-12 / fp)
    # zero mean of the Ricker: the antiderivative vanishes on both tails
    assert abs(float(inputs.ricker_integral(-10.0 * t0, fp))) < 1e-30
    assert abs(float(inputs.ricker_integral(12.0 * t0, fp))) < 1e-30
    assert abs(float(inputs.ricker_integral(t0, fp))) == 0.0


def test_injected_series():
    nt, dt, fp = 300, 8e-4, 10.0
    d32 = float(np.float32(dt))
    s_iso = inputs.source_series("iso", nt, dt, fp)
    s_ac = inputs.source_series("acoustic", nt, dt, fp)
    s_el = inputs.source_series("elastic", nt, dt, fp)
    assert s_iso.dtype == np.float32 and s_iso.shape == (nt,)
    n = np.arange(nt)
    assert np.array_equal(s_iso, inputs.ricker(n * d32, fp).astype(np.float32))
    assert np.array_equal(s_ac, s_el)
    # s[n] for the staggered schemes = integral of w up to (n + 1/2) dt (quadrature)
    for k in (0, 37, 150, 299):
        val, _ = quad(lambda s: float(inputs.ricker(s, fp)), -1.0, (k + 0.5) * d32, epsabs=1e-14,
                      epsrel=1e-12, limit=400)
        assert float(s_ac[k]) == pytest.approx(val, rel=1e-6, abs=1e-9)
    # the peak sample of the ISO series sits at t0 = 1.5 / fp
    assert n[np.argmax(s_iso)] * d32 == pytest.approx(1.5 / fp, abs=d32)
