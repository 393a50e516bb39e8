"""GPU <-> oracle parity of the NEXT-3 variant kernel through the C ABI (``-m gpu``).

Bidirectional halves (R22), probabilistic interpolation (R23) and the random / f-weighted
first fibre (R24) must match the oracle bit for bit: per half (nsteps, reason, end-point
bits), the polylines, the uint32 map and the connectivity matrix.  The variant kernel run
on the default semantics (PT_KERNEL_VARIANT) must match too.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import phantom
from tests.test_gpu_parity import (_targets, _threads, assert_parity, gpu_run, paths_equal, pt,  # noqa: F401
                                   tracker)

pytestmark = pytest.mark.gpu

REC = 1 | 2 | 4  # PT_REC_LEN | PT_REC_REASON | PT_REC_END


@pytest.mark.parametrize("bidir,interp,init", [
    (0, 0, 0), (1, 0, 0), (0, 1, 0), (0, 0, 1), (0, 0, 2), (1, 1, 2), (1, 1, 1),
])
def test_variants_dispersed_crossing(pt, tracker, bidir, interp, init):
    """Dispersed c2-shaped crossing (300 seeds x 400 particles, ragged CTA chunks): every
    half's (nsteps, reason, end) and the full map; (0,0,0) runs the variant kernel on the
    default semantics and must also equal the main kernel."""
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=300, particles_per_seed=400)
    w = w.replace(bidir=bidir, interp=interp, init_fibre=init)
    g = gpu_run(tracker, w, REC | pt.PT_KERNEL_VARIANT)
    r = oracle.track(w, threads=_threads())
    assert len(g["nsteps"]) == w.nparticles * (2 if bidir else 1)
    assert_parity(g, r)
    assert g["stats"]["total_steps"] == int(r["nsteps"].sum()) == int(g["map"].sum(dtype=np.uint64))
    assert g["stats"]["particles"] == w.nparticles
    if (bidir, interp, init) == (0, 0, 0):
        main = gpu_run(tracker, w, REC)
        assert_parity(main, r)


@pytest.mark.parametrize("half", [False, True])
@pytest.mark.parametrize("F", [1, 2, 3])
def test_variant_paths_bit_identical(pt, tracker, F, half):
    """Every point of every half's polyline, all variants on, F = 1..3, fp32 / fp16."""
    w = phantom.whole_brain(nx=40, ny=36, nz=24, semi=(17.0, 15.0, 10.0), nsamples=16, nfibres=F,
                            particles_per_seed=37)
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 120))
    w = w.replace(bidir=1, interp=1, init_fibre=2 if F > 1 else 1)
    if half:
        w = phantom.to_half(w)
    stride = 400
    g = gpu_run(tracker, w, REC | pt.PT_REC_PATHS, path_stride=stride)
    r = oracle.track(w, path_stride=stride, threads=_threads())
    assert_parity(g, r)
    assert paths_equal(g["paths"], r["paths"])


@pytest.mark.parametrize("mode", [0, 1])
def test_variant_connectivity_and_paper_mode(pt, tracker, mode):
    """NEXT-2 with bidirectional streamlines (union of the halves) and interpolation, in
    random-sample and paper mode (NEXT-1)."""
    import torch
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=150, particles_per_seed=200)
    w = w.replace(sample_mode=mode, bidir=1, interp=1)
    lab = _targets(w.volume.mask.shape, 40, seed=5)
    tracker.load_volume(w.volume)
    tracker.load_targets(lab, 40)
    m = tracker.track_workload(w, flags=REC | pt.PT_REC_CONN)
    torch.cuda.synchronize()
    g = tracker.get_paths()
    g["map"] = m.cpu().numpy().view(np.uint32)
    conn = tracker.connectivity().reshape(w.nseeds, 40)
    r = oracle.track(w, labels=lab, ntargets=40, threads=_threads())
    assert_parity(g, r)
    assert np.array_equal(conn.astype(np.uint64), r["conn"])
    assert conn.sum() > 500


def test_variant_closed_forms(pt, tracker):
    """The oracle pins' closed forms hold on the GPU too: bidirectional tube lengths
    (L+ + L- = 62 per particle) and the interpolated bent tube (23 or 24 steps)."""
    w = phantom.tube(particles_per_seed=64, seed_x=16).replace(bidir=1)
    g = gpu_run(tracker, w, REC)
    ns = g["nsteps"].astype(np.int64).reshape(-1, 2)
    assert np.all(ns.sum(1) == 62) and set(np.unique(ns)) == {30, 32}
    w = phantom.bent_tube(0.0, particles_per_seed=256).replace(interp=1)
    g = gpu_run(tracker, w, REC)
    assert set(np.unique(g["nsteps"].astype(np.int64))) == {16, 23, 24}
    assert_parity(g, oracle.track(w))


def test_variant_edge_cases(pt, tracker):
    """Seeds outside the volume / the mask, max_steps = 1, P = 1, nseeds = 0, and the
    argument errors of the variant flags."""
    import torch
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=20, particles_per_seed=33)
    seeds = w.seeds.copy()
    seeds[0] = (-4.0, 3.0, 2.0)
    seeds[1] = (0.5, 0.5, 0.5)
    for kw in (dict(), dict(max_steps=1), dict(particles_per_seed=1)):
        wv = w.replace(seeds=seeds, bidir=1, interp=1, init_fibre=1, **kw)
        g = gpu_run(tracker, wv, REC)
        assert_parity(g, oracle.track(wv))
    wv = w.replace(seeds=np.zeros((0, 3), np.float32), bidir=1)
    tracker.load_volume(wv.volume)
    m = tracker.track_workload(wv, flags=REC)
    torch.cuda.synchronize()
    assert int(m.sum().item()) == 0 and tracker.stats()["particles"] == 0
    for bad in (pt.PT_BIDIR | pt.PT_KERNEL_SIMPLE, pt.PT_INIT_RANDOM | pt.PT_INIT_FWEIGHT):
        with pytest.raises(pt.PtError) as e:
            tracker.track_workload(w, flags=bad)
        assert e.value.status == pt.PT_ERR_ARG


def test_variant_whole_brain_full_size_sampled(pt, tracker):
    """configs[2] at full size with bidirectional + interpolated tracking, in the launch
    configuration bench.py times for the variant line: global invariants at full size and
    2000 sampled particles (both halves) recomputed one by one by the oracle."""
    import torch
    w = phantom.config("c3").replace(bidir=1, interp=1)
    tracker.load_volume(w.volume)
    m = tracker.track_workload(w, flags=REC)
    torch.cuda.synchronize()
    st = tracker.stats()
    out = tracker.get_paths(on_device=True)
    nst = out["nsteps"].to(torch.int64)
    gm = m.cpu().numpy().view(np.uint32)
    assert nst.numel() == 2 * w.nparticles
    assert st["total_steps"] == int(nst.sum().item()) == int(gm.sum(dtype=np.uint64))
    assert np.all(gm[w.volume.mask == 0] == 0)
    rng = np.random.default_rng(2013)
    pick = np.sort(rng.choice(w.nparticles, 2000, replace=False))
    P = w.particles_per_seed
    rows = np.stack([2 * pick, 2 * pick + 1], 1).ravel()
    idx_t = torch.as_tensor(rows, device=out["nsteps"].device)
    g = {"nsteps": out["nsteps"][idx_t].cpu().numpy().view(np.uint16).astype(np.int64),
         "reason": out["reason"][idx_t].cpu().numpy(),
         "end": out["end"][idx_t].cpu().numpy()}
    rn, rr, re_ = [], [], []
    for li in pick:
        si, j = divmod(int(li), P)
        sub = w.replace(seeds=w.seeds[si:si + 1], seed_ids=w.ids()[si:si + 1])
        r = oracle.track(sub, j, j + 1, want_map=False)
        rn.extend(r["nsteps"])
        rr.extend(r["reason"])
        re_.extend(r["end"])
    assert np.array_equal(g["nsteps"], np.array(rn))
    assert np.array_equal(g["reason"], np.array(rr))
    assert np.array_equal(g["end"].view(np.uint32), np.array(re_).view(np.uint32))
