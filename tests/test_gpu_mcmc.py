"""GPU <-> oracle parity of the NEXT-4 MCMC sampler through the C ABI (``-m gpu``).

Parity bar: both sides follow C-MCMC in binary64 with the same operation
order, but exp/log/sin/cos come from different libraries (glibc vs CUDA, each within an
ulp or two) and the residual sum is a warp tree on the GPU, so a sample agrees to ~1e-13
relative; the bar is |gpu - oracle| <= 1e-9 (|oracle| + 1) per sample for every parameter.
A voxel whose chain took a different accept/reject decision (expected probability ~1e-14
per decision) would fail that bar; at most 1e-3 of the voxels may (expected: none).
"""
from __future__ import annotations

import os

import numpy as np
import pytest

import oracle
import phantom
from tests.test_gpu_parity import _threads, pt, tracker  # noqa: F401

pytestmark = pytest.mark.gpu

TOL = 1e-9


def _compare(g, r, nvox, max_frac=1e-3):
    """Per-voxel parity: every sample of every parameter within TOL (|o| + 1)."""
    g = np.asarray(g, np.float64)
    bad = np.abs(g - r) > TOL * (np.abs(r) + 1.0)
    per_vox = bad.reshape(bad.shape[0] * bad.shape[1], -1).any(0)
    nbad = int(per_vox.sum())
    assert nbad <= max(0, int(max_frac * nvox)), f"{nbad} of {nvox} voxels diverge"
    return nbad


def _run(tracker, d, **kw):
    import torch
    s, acc = tracker.mcmc(d, accepted=True, **kw)
    torch.cuda.synchronize()
    return s.cpu().numpy(), acc.cpu().numpy().view(np.uint32), tracker.mcmc_stats()


@pytest.mark.parametrize("N,ndirs,nb0", [(2, 60, 4), (1, 37, 4), (3, 96, 4), (2, 14, 2)])
def test_mcmc_parity_uniform(pt, tracker, N, ndirs, nb0):
    """Uniform voxels (noise differs per voxel), short chains, n = 64 / 41 / 100 / 16
    measurements (1-4 per lane, ragged last lanes), N = 1..3 fibres."""
    f = (0.45, 0.25, 0.1)[:N]
    v = ((1.0, 0.3, 0.2), (0.2, 1.0, -0.3), (0.1, -0.2, 1.0))[:N]
    d = phantom.dwi_uniform(nvox=96, f=f, v=v, ndirs=ndirs, nb0=nb0, gen_seed=30 + N,
                            burnin=60, nsamples=12, interval=2, adapt_every=10)
    g, gacc, st = _run(tracker, d)
    r = oracle.mcmc(d, threads=_threads())
    nbad = _compare(g, r["samples"], 96)
    if nbad == 0:
        assert np.array_equal(gacc, r["accepted"])
    assert st["voxels"] == 96 and st["mh_steps"] == 96 * d.loops * d.nparams
    assert st["accepted"] == int(gacc.sum())


@pytest.mark.parametrize("shells", [3, 40])
def test_mcmc_parity_multishell(pt, tracker, shells):
    """b-values on `shells` distinct shells: <= 8 shells take one e^{-b d'} per shell and
    proposal, more fall back to one per measurement; both must match the oracle."""
    rng = np.random.default_rng(shells)
    d = phantom.dwi_uniform(nvox=64, gen_seed=17, burnin=50, nsamples=10, interval=2, adapt_every=10)
    levels = np.round(rng.uniform(0.3, 3.0, shells), 3)
    b = d.bvals.copy()
    b[4:] = levels[np.arange(b.size - 4) % shells].astype(np.float32)
    d = d.replace(bvals=b)
    g, gacc, _ = _run(tracker, d)
    r = oracle.mcmc(d, threads=_threads())
    if _compare(g, r["samples"], 64) == 0:
        assert np.array_equal(gacc, r["accepted"])


def test_mcmc_parity_brain_small(pt, tracker):
    """Brain-shaped DWI (mask, mixed fibre configurations, automatic initial states)."""
    d = phantom.mcmc_config("m_small")
    g, gacc, st = _run(tracker, d)
    r = oracle.mcmc(d, threads=_threads())
    _compare(g, r["samples"], d.nvoxels)
    assert np.all(g[:, :, d.mask == 0] == 0)
    rate = gacc.reshape(d.nparams, -1)[:, d.mask.ravel() != 0] / d.loops
    assert 0.25 < rate.mean() < 0.5


def test_mcmc_fixed_and_init(pt, tracker):
    """M9 + caller-given initial state: only S0 and sigma free."""
    d = phantom.dwi_uniform(nvox=64, gen_seed=9, burnin=40, nsamples=20, interval=1, adapt_every=10)
    fixed = 0x1FF & ~((1 << 0) | (1 << 2))
    g, gacc, _ = _run(tracker, d, init=d.truth, fixed=fixed)
    r = oracle.mcmc(d, init=d.truth, fixed=fixed)
    _compare(g, r["samples"], 64)
    for k in range(9):
        if fixed >> k & 1:
            assert np.all(g[k] == d.truth[k][None])
            assert np.all(gacc[k] == 0)


def test_mcmc_full_size_sampled(pt, tracker):
    """configs m2 at full size (102x102x60, 402k valid voxels, 500 + 50 x 2 loops, the
    launch configuration bench.py times): 200 sampled voxels recomputed by the oracle."""
    d = phantom.mcmc_config("m2")
    g, gacc, st = _run(tracker, d)
    assert st["voxels"] == d.nvoxels
    idx = np.flatnonzero(d.mask.ravel())
    pick = np.sort(np.random.default_rng(7).choice(idx, 200, replace=False))
    r = oracle.mcmc(d, voxels=pick, threads=_threads())
    NP, S = d.nparams, d.nsamples
    gs = g.reshape(NP, S, -1)[:, :, pick]
    rs = r["samples"].reshape(NP, S, -1)[:, :, pick]
    _compare(gs, rs, 200, max_frac=0.005)
    rate = st["accepted"] / st["mh_steps"]
    assert 0.25 < rate < 0.5


def _to_volume_np(samples, mask, N):
    """(theta, phi) -> float32 unit vectors in numpy (test-side, for the oracle pipeline)."""
    S = samples.shape[1]
    dy = np.zeros((N, S) + mask.shape + (3,), np.float32)
    f = np.zeros((N, S) + mask.shape, np.float32)
    m = mask != 0
    for j in range(N):
        th, ph = samples[4 + 3 * j], samples[5 + 3 * j]
        v = np.stack([np.sin(th) * np.cos(ph), np.sin(th) * np.sin(ph), np.cos(th)], -1).astype(np.float32)
        dy[j] = np.where(m[None, ..., None], v, 0)
        f[j] = np.where(m[None], samples[3 + 3 * j].astype(np.float32), 0)
    return dy, f


def test_mcmc_to_tracking_pipeline(pt, tracker):
    """Fig. 1 end to end: GPU samples -> pt_mcmc_to_volume -> pt_load_samples -> pt_track
    versus oracle samples -> numpy conversion -> oracle tracker.  The conversion differs by
    at most 1 ulp of float32 between libraries, so the tracking comparison uses the north
    star's divergence tolerance (<= 1e-4 ... here <= 1e-3 of a small run)."""
    import torch
    d = phantom.mcmc_config("m_small")
    s, _ = tracker.mcmc(d)
    dy, f = tracker.mcmc_to_volume(s, d.mask, d.nfibres)
    torch.cuda.synchronize()
    r = oracle.mcmc(d, threads=_threads())
    ody, of = _to_volume_np(r["samples"], d.mask, d.nfibres)
    gdy, gf = dy.cpu().numpy(), f.cpu().numpy()
    ulp = np.abs(gdy.view(np.int32).astype(np.int64) - ody.view(np.int32).astype(np.int64))
    assert ulp.max() <= 2 and np.mean(ulp > 0) < 0.05
    assert np.array_equal(gf, of)
    vol = phantom.Volume(d.nx, d.ny, d.nz, d.nsamples, d.nfibres, ody, of, d.mask)
    seeds = phantom._centres(np.argwhere(d.mask)[::7, ::-1])
    w = phantom.Workload("mcmc_pipeline", vol, seeds, None, particles_per_seed=50, curv_thr=0.2)
    tracker.load_samples(dy, f, torch.as_tensor(d.mask, device="cuda"), d.nsamples, d.nfibres)
    flags = pt.PT_REC_LEN | pt.PT_REC_REASON | pt.PT_REC_END
    m = tracker.track_workload(w, flags=flags)
    torch.cuda.synchronize()
    g = tracker.get_paths()
    ref = oracle.track(w, threads=_threads())
    div = (g["nsteps"].astype(np.int64) != ref["nsteps"]) | (g["reason"] != ref["reason"]) | \
        np.any(g["end"].view(np.uint32) != ref["end"].view(np.uint32), axis=1)
    assert div.mean() <= 1e-3 + 1.0 / len(div), div.mean()
    gm = m.cpu().numpy().view(np.uint32).astype(np.int64)
    assert np.abs(gm - ref["map"].astype(np.int64)).sum() <= 1e-3 * ref["map"].sum() + 50
    assert ref["nsteps"].mean() > 3


def test_mcmc_errors(pt, tracker):
    d = phantom.dwi_uniform(nvox=4)
    with pytest.raises(pt.PtError) as e:
        tracker.mcmc(d.replace(nfibres=4))
    assert e.value.status == pt.PT_ERR_ARG
    with pytest.raises(pt.PtError) as e:
        tracker.mcmc(d.replace(interval=0))
    assert e.value.status == pt.PT_ERR_ARG
    big = phantom.dwi_uniform(nvox=2, ndirs=140)
    with pytest.raises(pt.PtError) as e:
        tracker.mcmc(big)
    assert e.value.status == pt.PT_ERR_ARG
    empty = d.replace(mask=np.zeros_like(d.mask))
    s, _ = tracker.mcmc(empty)
    assert float(s.abs().sum().item()) == 0.0 and tracker.mcmc_stats()["voxels"] == 0
