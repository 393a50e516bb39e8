"""The method's tie and degenerate cases on EVERY tracking kernel (``-m gpu``), element by
element against the oracle.  The rules come from the paper where it speaks and from the
readings where it is silent: the angle test at exactly the threshold (R4),
fibre eligibility f == fib_thr (R7), equal |dot| between fibres (R8), a zero dot
with a negative threshold (R9), no eligible fibre (R7), the T-junction (C-pin-7),
isotropic samples (C-pin-9) and mirror symmetry (C-pin-8).  The dispersed random phantoms
of the other suites essentially never produce an exact tie, so these phantoms are the ones
that reach the tie branches.

Kernels: the persistent round kernel with per-particle outputs (OUT), the SAME kernel as
bench.py times (flags = 0: no outputs, compile-time bricked layout) compared on the map, the
no-refill ablation, the segmented-relaunch ablation, the variant instantiation on the
default semantics, and the unique-map instantiation (step map via its own counters)."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
import phantom

pytestmark = pytest.mark.gpu

KERNELS = ["main", "bench", "simple", "segmented", "variant"]


@pytest.fixture(scope="module")
def pt():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_ipps_xuzwrwxgxy12_b200 as m
    m.build()
    return m


@pytest.fixture(scope="module")
def tracker(pt):
    t = pt.Tracker(0)
    yield t
    t.close()


def _run(pt, tr, w, kernel):
    import torch
    rec = pt.PT_REC_LEN | pt.PT_REC_REASON | pt.PT_REC_END
    flags = {"main": rec, "bench": 0, "simple": rec | pt.PT_KERNEL_SIMPLE,
             "segmented": rec | pt.PT_KERNEL_SEGMENTED, "variant": rec | pt.PT_KERNEL_VARIANT}[kernel]
    tr.load_volume(w.volume)
    m = tr.track_workload(w, flags=flags)
    torch.cuda.synchronize()
    out = tr.get_paths() if flags & rec else {}
    out["map"] = m.cpu().numpy().view(np.uint32)
    out["stats"] = tr.stats()
    return out


def _check(pt, tr, w, kernel, r=None):
    r = oracle.track(w) if r is None else r
    g = _run(pt, tr, w, kernel)
    if "nsteps" in g:
        assert np.array_equal(g["nsteps"].astype(np.int64), r["nsteps"].astype(np.int64)), kernel
        assert np.array_equal(g["reason"], r["reason"]), kernel
        assert np.array_equal(g["end"].view(np.uint32), r["end"].view(np.uint32)), kernel
    assert np.array_equal(g["map"].astype(np.uint64), r["map"]), kernel
    assert g["stats"]["total_steps"] == int(r["nsteps"].sum())
    return g, r


def _cs():
    c = np.float32(0.6)
    return c, np.float32(math.sqrt(1 - float(c) ** 2))


CASES = {
    # R4: the fp32 dot equals the threshold exactly -> CURV; one ulp above -> continues
    "bent_at_threshold": lambda: phantom.bent_tube(0.2, curv_thr=0.2, particles_per_seed=64),
    "bent_above_threshold": lambda: phantom.bent_tube(float(np.nextafter(np.float32(0.2), np.float32(1))),
                                                      curv_thr=0.2, particles_per_seed=64),
    # R8: equal |dot| -> the lower index wins; with opposite signs the winner is flipped (R9)
    "fork_equal_dot": lambda: phantom.fork([((_cs()[0], _cs()[1], 0), 0.5), ((_cs()[0], -_cs()[1], 0), 0.5)]),
    "fork_equal_dot_opposite": lambda: phantom.fork([((-_cs()[0], _cs()[1], 0), 0.5),
                                                     ((_cs()[0], -_cs()[1], 0), 0.5)]),
    # R7: f == fib_thr is not eligible; one ulp above is
    "fork_f_at_thr": lambda: phantom.fork([((1, 0, 0), np.float32(0.01)), ((_cs()[0], -_cs()[1], 0), 0.5)],
                                          fib_thr=0.01),
    "fork_f_above_thr": lambda: phantom.fork([((1, 0, 0), np.nextafter(np.float32(0.01), np.float32(1))),
                                              ((_cs()[0], -_cs()[1], 0), 0.5)], fib_thr=0.01),
    # R7: no eligible fibre -> fibre 0, never a termination on f
    "fork_none_eligible": lambda: phantom.fork([((1, 0, 0), 0.0), ((0, 1, 0), 0.0)]),
    # C-pin-7 and R9 (zero dot with a negative threshold: sign -1)
    "t_junction": lambda: phantom.t_junction(x_j=40, seed_xs=(20, 30), particles_per_seed=100),
    "t_junction_negative_thr": lambda: phantom.t_junction(x_j=40, seed_xs=(30,), particles_per_seed=64,
                                                          curv_thr=-0.5),
    # C-pin-9: isotropic samples, geometric lengths (small)
    "isotropic": lambda: phantom.isotropic(n=24, nsamples=512, nfibres=2, nseeds=4, particles_per_seed=2000),
    "isotropic_f3": lambda: phantom.isotropic(n=20, nsamples=256, nfibres=3, nseeds=3, particles_per_seed=1000,
                                              curv_thr=0.5),
}


@pytest.mark.parametrize("kernel", KERNELS)
@pytest.mark.parametrize("case", sorted(CASES))
def test_tie_case(pt, tracker, case, kernel):
    _check(pt, tracker, CASES[case](), kernel)


@pytest.mark.parametrize("kernel", KERNELS)
def test_mirror_symmetry(pt, tracker, kernel):
    """C-pin-8 on the GPU: mirrored phantom with the same ids -> the maps mirror bit-exactly
    and each side equals the oracle."""
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=40, particles_per_seed=50, nsamples=20)
    m = phantom.mirror_x(w)
    ga, _ = _check(pt, tracker, w, kernel)
    gb, _ = _check(pt, tracker, m, kernel)
    assert np.array_equal(ga["map"][:, :, ::-1], gb["map"])


@pytest.mark.parametrize("kernel", ["main", "bench", "simple", "segmented", "variant"])
def test_half_precision_ties(pt, tracker, kernel):
    """The bent tube at threshold with fp16 records: the threshold value is a half (0.25),
    so the fp32 dot of the decoded half equals it exactly."""
    w = phantom.to_half(phantom.bent_tube(0.25, curv_thr=0.25, particles_per_seed=64))
    _check(pt, tracker, w, kernel)


def test_nan_and_far_seeds(pt, tracker):
    """Non-finite and far-away seeds are outside the volume (R12): 0 steps, MASK, on every
    kernel; the rest of the call is unaffected."""
    w = phantom.crossing(sigma=0.15, nseeds=10, particles_per_seed=16)
    bad = np.array([[np.nan, 3.0, 3.0], [np.inf, 1, 1], [-np.inf, 1, 1], [1e30, 1, 1], [3.0, 3.0, -1e9]],
                   np.float32)
    ww = w.replace(seeds=np.concatenate([w.seeds, bad]))
    r = oracle.track(ww)
    for kernel in KERNELS:
        g = _run(pt, tracker, ww, kernel)
        assert np.array_equal(g["map"].astype(np.uint64), r["map"])
        if "nsteps" in g:
            assert np.array_equal(g["nsteps"].astype(np.int64), r["nsteps"].astype(np.int64))
            assert np.array_equal(g["reason"], r["reason"])
            n_bad = len(bad) * w.particles_per_seed
            assert np.all(g["nsteps"][-n_bad:] == 0) and np.all(g["reason"][-n_bad:] == oracle.END_MASK)
