"""Pins of the NEXT-4 MCMC oracle (CPU only, readings M1-M9).

Expectations come from closed forms of Eq. 1, known Gaussian / inverse-gamma posteriors
(parameters held fixed with M9 so that the remaining conditional posterior is analytic),
the KS law of the Box-Muller draws, the paper's acceptance band, recovery of the
generating parameters at high SNR, and an independent pure-Python transcription
(tests/bruteforce_mcmc.py) -- never from the oracle itself.
"""
from __future__ import annotations

import math

import numpy as np
import pytest
from scipy import stats

import oracle
import phantom
from tests import bruteforce_mcmc as bf

S0_, D_, SIG_, F1, TH1, PH1, F2, TH2, PH2 = range(9)
ALL9 = (1 << 9) - 1


def _free(*ks):
    return ALL9 & ~sum(1 << k for k in ks)


# ----------------------------------------------------------------------------- Eq. 1

def test_signal_closed_forms():
    """Eq. 1 special cases: b = 0 -> S0; f = 0 -> S0 e^{-bd}; a single stick
    along r -> S0 e^{-bd}; a stick perpendicular to r -> S0 (f = 1)."""
    bvals, bvecs = phantom.gradient_scheme(30, 2, 1.3)
    w = np.array([900.0, 0.8, 10.0, 0.0, 0.4, 1.1, 0.0, 2.0, -0.3])
    mu = oracle.mcmc_signal(2, w, bvals, bvecs)
    expect = 900.0 * np.exp(-bvals.astype(np.float64) * 0.8)
    assert np.allclose(mu, expect, rtol=1e-15, atol=0)
    assert np.all(mu[:2] == 900.0)
    # one fibre, f = 1, v = e_z; r = e_z -> S0 e^{-bd}; r = e_x -> S0
    r = np.array([[0, 0, 1], [1, 0, 0], [0, 1, 0]], np.float32)
    b = np.array([1.0, 1.0, 2.0], np.float32)
    mu = oracle.mcmc_signal(1, [500.0, 1.5, 1.0, 1.0, 0.0, 0.0], b, r)
    assert mu[0] == pytest.approx(500.0 * math.exp(-1.5), rel=1e-15)
    assert mu[1] == pytest.approx(500.0, rel=1e-15) and mu[2] == pytest.approx(500.0, rel=1e-15)


@pytest.mark.parametrize("N", [1, 2, 3])
def test_signal_matches_generator_forward_model(N):
    """Eq. 1 against the generator's independent vectorised numpy forward model."""
    rng = np.random.default_rng(N)
    bvals, bvecs = phantom.gradient_scheme(60, 4, 1.0)
    for _ in range(20):
        f = rng.dirichlet(np.ones(N + 1))[:N] * 0.9
        th = rng.uniform(0, math.pi, N)
        ph = rng.uniform(-math.pi, math.pi, N)
        S0, d = rng.uniform(500, 1500), rng.uniform(0.3, 2.0)
        w = [S0, d, 5.0]
        v = []
        for j in range(N):
            w += [f[j], th[j], ph[j]]
            v.append([[math.sin(th[j]) * math.cos(ph[j]), math.sin(th[j]) * math.sin(ph[j]), math.cos(th[j])]])
        mu = oracle.mcmc_signal(N, w, bvals, bvecs)
        ref = phantom._forward(np.array([S0]), np.array([d]), f[:, None], np.array(v), bvals, bvecs)[:, 0]
        assert np.allclose(mu, ref, rtol=1e-13, atol=0)


# ----------------------------------------------------------------------------- draws (M6)

def test_draws_are_standard_normal_and_uniform():
    """M6: Box-Muller Gaussians N(0,1) and uniforms (KS), over (loop, voxel, k)."""
    zs, us = [], []
    for t in range(400):
        for v in (0, 7, 123456):
            for k in range(9):
                z, lu = oracle.mcmc_draw(99, t, v, k)
                zs.append(z)
                us.append(math.exp(lu))
    assert stats.kstest(zs, "norm").pvalue > 1e-4
    assert stats.kstest(us, "uniform").pvalue > 1e-4
    assert abs(np.mean(zs)) < 0.03 and abs(np.var(zs) - 1) < 0.05


def test_draw_counter_layout():
    """M6 contract: counter {loop, voxel, k, "MCMC"}, key = seed; u1 = (w0 + 1/2) 2^-32,
    u2 = w1 2^-32, u3 = (w2 + 1/2) 2^-32 (Philox pinned by the Random123 answers)."""
    for (seed, t, v, k) in [(0, 0, 0, 0), (2**40 + 5, 17, 99, 8), (123, 2**31, 2**32 - 1, 3)]:
        z, lu = oracle.mcmc_draw(seed, t, v, k)
        zb, lub = bf.draw(seed, t, v, k)
        assert z == pytest.approx(zb, rel=1e-14, abs=1e-15) and lu == pytest.approx(lub, rel=1e-14)


# ----------------------------------------------------------------------------- MH (known posteriors)

def _uniform(nvox=100, **kw):
    base = dict(burnin=200, nsamples=400, interval=5, adapt_every=50, rng_seed=314)
    base.update(kw)
    return phantom.dwi_uniform(nvox=nvox, gen_seed=11, **base)


def _design(d):
    """A_i = (1 - f1 - f2) e0 + f1 e1 + f2 e2 at the truth (so mu = S0 A); per voxel."""
    t = d.truth.reshape(9, -1)[:, 0]
    return oracle.mcmc_signal(2, np.r_[1.0, t[1:]], d.bvals, d.bvecs)


def test_s0_conditional_posterior_is_gaussian():
    """M9: everything but S0 fixed at the truth: mu = S0 A (flat prior) => S0 | y ~
    N(sum y A / sum A^2, sigma^2 / sum A^2).  Pooled standardised samples: mean 0, var 1."""
    d = _uniform()
    A = _design(d)
    sig = d.truth.reshape(9, -1)[SIG_, 0]
    y = d.dwi.reshape(d.nmeas, -1).astype(np.float64)
    m = (A[:, None] * y).sum(0) / (A * A).sum()
    s = sig / math.sqrt((A * A).sum())
    r = oracle.mcmc(d, init=d.truth, fixed=_free(S0_))
    smp = r["samples"].reshape(9, d.nsamples, -1)
    zz = (smp[S0_] - m[None, :]) / s
    assert abs(zz.mean()) < 0.06, zz.mean()
    assert 0.9 < zz.var() < 1.1, zz.var()
    for k in range(1, 9):   # fixed parameters never move
        assert np.all(smp[k] == d.truth.reshape(9, -1)[k][None, :])


def test_sigma_conditional_posterior_is_inverse_gamma():
    """M2/M3/M9: only sigma free: p(sigma | y) ~ sigma^-(n+1) exp(-SSE / 2 sigma^2) =>
    SSE / sigma^2 ~ chi^2_n (mean n, variance 2n)."""
    d = _uniform()
    t = d.truth.reshape(9, -1)
    y = d.dwi.reshape(d.nmeas, -1).astype(np.float64)
    mu = oracle.mcmc_signal(2, t[:, 0], d.bvals, d.bvecs)
    sse = ((y - mu[:, None]) ** 2).sum(0)
    r = oracle.mcmc(d, init=d.truth, fixed=_free(SIG_))
    smp = r["samples"].reshape(9, d.nsamples, -1)[SIG_]
    q = sse[None, :] / smp ** 2
    n = d.nmeas
    assert abs(q.mean() - n) < 0.03 * n, q.mean()
    assert 0.85 * 2 * n < q.var() < 1.15 * 2 * n, q.var()


def test_f1_conditional_posterior_is_gaussian():
    """M1-M3: only f1 free: mu = S0 [e0 + f1 (e1 - e0) + f2 (e2 - e0)] is linear in f1 =>
    Gaussian posterior (far from the support bounds).  Pins the (1 - sum f) term of Eq. 1."""
    d = _uniform()
    t = d.truth.reshape(9, -1)[:, 0]
    e = [oracle.mcmc_signal(2, np.r_[t[0], t[1:3], fz], d.bvals, d.bvecs)
         for fz in ([0, t[TH1], t[PH1], 0, t[TH2], t[PH2]],
                    [1, t[TH1], t[PH1], 0, t[TH2], t[PH2]],
                    [0, t[TH1], t[PH1], 1, t[TH2], t[PH2]])]
    B = e[1] - e[0]
    mu0 = e[0] + t[F2] * (e[2] - e[0])
    y = d.dwi.reshape(d.nmeas, -1).astype(np.float64)
    m = (B[:, None] * (y - mu0[:, None])).sum(0) / (B * B).sum()
    s = t[SIG_] / math.sqrt((B * B).sum())
    r = oracle.mcmc(d, init=d.truth, fixed=_free(F1))
    zz = (r["samples"].reshape(9, d.nsamples, -1)[F1] - m[None, :]) / s
    assert abs(zz.mean()) < 0.06 and 0.88 < zz.var() < 1.12, (zz.mean(), zz.var())


def test_acceptance_rates_in_the_papers_band():
    """the adapted proposals keep every acceptance rate between 25% and 50%."""
    d = phantom.dwi_uniform(nvox=24, gen_seed=3)
    r = oracle.mcmc(d)
    rate = r["accepted"].reshape(9, -1) / d.loops
    assert np.all(rate > 0.25) and np.all(rate < 0.5), rate.mean(1)


def _axis_angle(th, ph, th0, ph0):
    v = np.stack([np.sin(th) * np.cos(ph), np.sin(th) * np.sin(ph), np.cos(th)], -1)
    v0 = np.array([math.sin(th0) * math.cos(ph0), math.sin(th0) * math.sin(ph0), math.cos(th0)])
    T = np.einsum("...i,...j->...ij", v, v).mean(axis=0)   # mean dyadic over samples
    _, U = np.linalg.eigh(T)
    return math.degrees(math.acos(min(1.0, abs(float(U[:, -1] @ v0)))))


def test_recovers_generating_parameters_at_high_snr():
    """Posterior means at SNR 400 from the automatic initial state (M7): S0 within 1%,
    d within 3%, sigma within 20%, f within 0.03, fibre axes within 3 degrees."""
    d = phantom.dwi_uniform(nvox=6, snr=400.0, gen_seed=8, f=(0.45, 0.25),
                            v=((0.8, 0.6, 0.0), (0.0, 0.3, 0.95)))
    r = oracle.mcmc(d)
    s = r["samples"].reshape(9, d.nsamples, -1)
    t = d.truth.reshape(9, -1)
    for vox in range(6):
        assert abs(s[S0_, :, vox].mean() / t[S0_, vox] - 1) < 0.01
        assert abs(s[D_, :, vox].mean() / t[D_, vox] - 1) < 0.03
        assert abs(s[SIG_, :, vox].mean() / t[SIG_, vox] - 1) < 0.2
        assert abs(s[F1, :, vox].mean() - t[F1, vox]) < 0.03
        assert abs(s[F2, :, vox].mean() - t[F2, vox]) < 0.03
        assert _axis_angle(s[TH1, :, vox], s[PH1, :, vox], t[TH1, vox], t[PH1, vox]) < 3.0
        assert _axis_angle(s[TH2, :, vox], s[PH2, :, vox], t[TH2, vox], t[PH2, vox]) < 3.0


# ----------------------------------------------------------------------------- bookkeeping + brute force

def _init_state(d, voxel):
    """M7 restated: S0 = mean b=0 signal; d = -ln(mean DW / S0) / mean b; fibre j = DW
    direction of the smallest signal with |r.v_k| < 1/2 for earlier fibres; f = 0.3, 0.1;
    sigma = max(RMS residual, 1e-3 S0)."""
    V = d.nx * d.ny * d.nz
    y = [float(d.dwi.reshape(-1, V)[i, voxel]) for i in range(d.nmeas)]
    b0 = [yi for yi, b in zip(y, d.bvals) if b == 0]
    dw = [(yi, float(b), i) for i, (yi, b) in enumerate(zip(y, d.bvals)) if b != 0]
    S0 = sum(b0) / len(b0)
    dd = -math.log((sum(x[0] for x in dw) / len(dw)) / S0) / (sum(x[1] for x in dw) / len(dw))
    picks = []
    for j in range(d.nfibres):
        best = None
        for yi, _, i in dw:
            r = d.bvecs[i].astype(np.float64)
            if all(abs(float(r @ d.bvecs[m].astype(np.float64))) < 0.5 for m in picks):
                if best is None or yi < best[0]:
                    best = (yi, i)
        picks.append(best[1])
    w = [S0, dd, 1.0]
    for j, i in enumerate(picks):
        r = d.bvecs[i].astype(np.float64)
        w += [0.3 if j == 0 else 0.1, math.acos(max(-1.0, min(1.0, r[2]))), math.atan2(r[1], r[0])]
    mu = bf.signal(d.nfibres, w, d.bvals, d.bvecs)
    rms = math.sqrt(sum((a - b) ** 2 for a, b in zip(y, mu)) / len(y))
    w[2] = max(rms, 1e-3 * S0)
    return w


@pytest.mark.parametrize("N", [1, 2, 3])
def test_bruteforce_chains(N):
    """C-pin-11 for NEXT-4: the pure-Python transcription, started from the restated
    automatic initial state, reproduces the oracle's samples and acceptance counts."""
    f = (0.5, 0.3, 0.1)[:N]
    v = ((1.0, 0.2, 0.1), (0.1, 1.0, -0.3), (0.2, -0.1, 1.0))[:N]
    d = phantom.dwi_uniform(nvox=3, f=f, v=v, gen_seed=20 + N, burnin=30, nsamples=8,
                            interval=3, adapt_every=7)
    r = oracle.mcmc(d)
    NP = 3 + 3 * N
    smp = r["samples"].reshape(NP, d.nsamples, -1)
    for vox in range(3):
        init = _init_state(d, vox)
        out, tot = bf.chain(d, vox, init)
        assert np.allclose(np.array(out).T, smp[:, :, vox], rtol=1e-12, atol=1e-12)
        assert list(r["accepted"].reshape(NP, -1)[:, vox]) == tot


def test_first_mh_step_by_hand():
    """One loop, one free parameter (S0), burn-in 0, L = 1: the single sample is S0 + 0.01 S0 z
    iff log u < lp' - lp, else S0 (M6, M8)."""
    d = phantom.dwi_uniform(nvox=40, gen_seed=2, burnin=0, nsamples=1, interval=1)
    r = oracle.mcmc(d, init=d.truth, fixed=_free(S0_))
    got = r["samples"].reshape(9, -1)[S0_]
    t = d.truth.reshape(9, -1)
    moved = 0
    for vox in range(40):
        w = list(t[:, vox])
        y = [float(x) for x in d.dwi.reshape(d.nmeas, -1)[:, vox]]
        z, lu = bf.draw(d.rng_seed, 0, vox, S0_)
        wn = list(w)
        wn[0] = w[0] + 0.01 * w[0] * z
        acc = lu < bf.log_post(2, wn, y, d.bvals, d.bvecs) - bf.log_post(2, w, y, d.bvals, d.bvecs)
        assert got[vox] == pytest.approx(wn[0] if acc else w[0], rel=1e-14)
        moved += acc
    assert 0 < moved < 40


def test_sample_schedule_and_sharding():
    """sample s is the state after loop burnin + (s+1) L - 1 (a run with that
    burn-in and one sample per loop reproduces it); voxel-range threading is exact."""
    d = phantom.dwi_uniform(nvox=5, gen_seed=6, burnin=20, nsamples=4, interval=3, adapt_every=10)
    r = oracle.mcmc(d)["samples"]
    for s in range(4):
        e = oracle.mcmc(d.replace(burnin=20 + (s + 1) * 3 - 1, nsamples=1, interval=1))["samples"]
        assert np.array_equal(e[:, 0], r[:, s])
    r3 = oracle.mcmc(d, threads=3)["samples"]
    assert np.array_equal(r3, r)
    sub = oracle.mcmc(d, voxels=np.array([1, 3]))["samples"].reshape(9, 4, -1)
    assert np.array_equal(sub[:, :, [1, 3]], r.reshape(9, 4, -1)[:, :, [1, 3]])
    assert np.all(sub[:, :, [0, 2, 4]] == 0)


def test_support_bounds_are_enforced():
    """M3: proposals outside f_j >= 0, sum f <= 1 (Eq. 1 needs 1 - sum f >= 0) are rejected:
    with the truth on a bound, the free f1 piles up against it and never crosses."""
    d = phantom.dwi_uniform(nvox=40, f=(0.39, 0.6), gen_seed=12, burnin=100, nsamples=200,
                            interval=2, snr=60.0)
    s = oracle.mcmc(d, init=d.truth, fixed=_free(F1))["samples"].reshape(9, d.nsamples, -1)
    assert np.all(s[F1] + s[F2] <= 1.0) and s[F1].max() > 0.399
    d = phantom.dwi_uniform(nvox=40, f=(0.003, 0.5), gen_seed=13, burnin=100, nsamples=200,
                            interval=2, snr=60.0)
    s = oracle.mcmc(d, init=d.truth, fixed=_free(F1))["samples"].reshape(9, d.nsamples, -1)
    assert np.all(s[F1] >= 0.0) and s[F1].min() < 0.001
