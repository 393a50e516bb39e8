"""GPU parity of the speculative-gather kernel (``PT_KERNEL_SPEC``, csrc/pt_spec.cu;
DESIGN.md §13): a second record gather at the extrapolated next voxel, used only when it
is exactly the record the sequential algorithm (C-ALG) reads, so every output must be
bit-identical to the oracle.  Same bar and helpers as test_gpu_parity.py."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import phantom
from tests.test_gpu_parity import _targets, _threads, assert_parity, gpu_run, paths_equal, pt, tracker  # noqa: F401

pytestmark = pytest.mark.gpu


def _rec(pt):
    return pt.PT_REC_LEN | pt.PT_REC_REASON | pt.PT_REC_END | pt.PT_KERNEL_SPEC


def test_spec_c1_c2_full(pt, tracker):
    for cfg in ("c1", "c2", "c2_dispersed"):
        w = phantom.config(cfg)
        g = gpu_run(tracker, w, _rec(pt))
        r = oracle.track(w, threads=_threads())
        assert_parity(g, r)
        assert g["stats"]["total_steps"] == int(r["nsteps"].sum())
    # dispersed crossing: most second steps come from the speculative record
    assert g["stats"]["spec_hits"] > 0.3 * g["stats"]["total_steps"]


@pytest.mark.parametrize("half", [False, True])
@pytest.mark.parametrize("F", [1, 2, 3])
def test_spec_paths_bit_identical(pt, tracker, F, half):
    w = phantom.whole_brain(nx=40, ny=36, nz=24, semi=(17.0, 15.0, 10.0), nsamples=16, nfibres=F,
                            particles_per_seed=37)
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 150))
    if half:
        w = phantom.to_half(w)
    g = gpu_run(tracker, w, _rec(pt) | pt.PT_REC_PATHS, path_stride=512)
    r = oracle.track(w, path_stride=512, threads=_threads())
    assert_parity(g, r)
    assert paths_equal(g["paths"], r["paths"])


@pytest.mark.parametrize("half", [False, True])
def test_spec_paper_mode(pt, tracker, half):
    w = phantom.paper_dataset(1, 0.2, 0.8)
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 1500))
    if half:
        w = phantom.to_half(w)
    g = gpu_run(tracker, w, _rec(pt) | pt.PT_REC_PATHS, path_stride=256)
    r = oracle.track(w, path_stride=256, threads=_threads())
    assert_parity(g, r)
    assert paths_equal(g["paths"], r["paths"])


def test_spec_connectivity_and_max_steps(pt, tracker):
    import torch
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=200, particles_per_seed=300)
    lab = _targets(w.volume.mask.shape, 64, seed=7)
    tracker.load_volume(w.volume)
    tracker.load_targets(lab, 64)
    m = tracker.track_workload(w, flags=_rec(pt) | pt.PT_REC_CONN)
    torch.cuda.synchronize()
    g = tracker.get_paths()
    g["map"] = m.cpu().numpy().view(np.uint32)
    conn = tracker.connectivity().reshape(w.nseeds, 64)
    r = oracle.track(w, labels=lab, ntargets=64, threads=_threads())
    assert_parity(g, r)
    assert np.array_equal(conn.astype(np.uint64), r["conn"])
    # MAXLEN reached inside a two-step iteration (every max_steps parity)
    for ms in (1, 2, 3, 4, 7):
        wm = w.replace(max_steps=ms)
        g = gpu_run(tracker, wm, _rec(pt))
        r = oracle.track(wm, threads=_threads())
        assert_parity(g, r)


def test_spec_whole_brain_sampled(pt, tracker):
    """c3 shape (full volume), every 400th WM seed x 5000: every particle and the map."""
    w = phantom.wm_seeds(phantom.config("c3"), every=400)
    g = gpu_run(tracker, w, _rec(pt))
    r = oracle.track(w, threads=_threads())
    assert_parity(g, r)


def test_spec_rejects_other_kernels(pt, tracker):
    w = phantom.config("c1")
    tracker.load_volume(w.volume)
    for bad in (pt.PT_KERNEL_SIMPLE, pt.PT_KERNEL_SEGMENTED, pt.PT_BIDIR, pt.PT_KERNEL_VARIANT):
        with pytest.raises(pt.PtError):
            tracker.track_workload(w, flags=pt.PT_KERNEL_SPEC | bad)
