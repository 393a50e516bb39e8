"""Pins of the NEXT-3 oracle variants (CPU only): bidirectional streamlines (R22),
probabilistic interpolation of the sampled voxel (R23, "Interpolation()" P:L175) and the
random / f-weighted first fibre (R24).  Every expectation below comes from a closed form,
from Philox words alone (pinned by the Random123 known answers, C-pin-1), from binomial
statistics, or from the independent numpy tracker (tests/bruteforce.py) -- never from the
oracle itself.
"""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
import phantom
from tests import bruteforce
from tests.test_oracle_pins import _exact_path, _signs

_M = 0xFFFFFFFF


def _words(w, pid, block, stream):
    key = (w.rng_seed & _M, w.rng_seed >> 32)
    return [int(x) for x in oracle.philox([block, pid & _M, pid >> 32, stream], key)]


def _pids(w):
    P = w.particles_per_seed
    return [int(sid) * P + j for sid in w.ids() for j in range(P)]


def _binomial_ok(k, n, p, z=4.5):
    sd = math.sqrt(n * p * (1 - p))
    return abs(k - n * p) <= z * sd + 1


# ----------------------------------------------------------------------------- R22 bidirectional

def test_bidir_tube_closed_form():
    """Zero-dispersion tube (C-pin-5 geometry): half 0 runs L_sign, half 1 the opposite
    direction L_-sign, both end MASK; the map is the sum of both halves' exact paths."""
    N, xs = 32, 16
    w = phantom.tube(particles_per_seed=40, seed_x=xs).replace(bidir=1)
    r = oracle.track(w)
    sg = _signs(w)
    Lp, Lm = 30, 32                 # c = 16, xs = 16, full tube (hand-derived, C-pin-5)
    ns = r["nsteps"].reshape(-1, 2)
    assert np.array_equal(ns[:, 0], np.where(sg > 0, Lp, Lm))
    assert np.array_equal(ns[:, 1], np.where(sg > 0, Lm, Lp))
    assert np.all(r["reason"] == oracle.END_MASK)
    end = r["end"].reshape(-1, 2, 3)
    for h, s in ((0, sg), (1, -sg)):
        L = np.where(s > 0, Lp, Lm)
        ex = (np.float32(xs) + np.float32(0.5) + np.float32(0.5) * s * L).astype(np.float32)
        assert np.array_equal(end[:, h, 0], ex)
    m = np.zeros_like(r["map"])
    seeds = np.repeat(w.seeds, w.particles_per_seed, 0)
    for i, s in enumerate(sg):
        sy, sz = int(seeds[i, 1]), int(seeds[i, 2])
        for h, sh in ((0, s), (1, -s)):
            for vx in _exact_path(N, xs, int(sh), int(ns[i, h])):
                m[sz, sy, vx] += 1
    assert np.array_equal(r["map"], m)
    assert int(r["map"].sum()) == int(r["nsteps"].sum())


def test_bidir_half0_is_the_one_directional_particle():
    """Half 0 draws from stream 0 exactly like the one-directional particle (R16, R22)."""
    w = phantom.whole_brain(nx=24, ny=24, nz=16, semi=(10.0, 10.5, 6.5), nsamples=12,
                            particles_per_seed=20)
    one = oracle.track(w, path_stride=64)
    two = oracle.track(w.replace(bidir=1), path_stride=64)
    for k in ("nsteps", "reason", "end", "paths"):
        a = one[k]
        b = np.ascontiguousarray(two[k].reshape((-1, 2) + a.shape[1:])[:, 0])
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8)), k
    assert int(two["map"].sum()) == int(two["nsteps"].sum())
    assert int(two["map"].sum()) > int(one["map"].sum())


def _parity_box(S=4, P=200, nx=24, ny=24, nz=8):
    """F = 1, every voxel inside; sample s points along x (s even) or y (s odd)."""
    dy = np.zeros((1, S, nz, ny, nx, 3), np.float32)
    dy[0, 0::2, ..., 0] = 1.0
    dy[0, 1::2, ..., 1] = 1.0
    f = np.ones((1, S, nz, ny, nx), np.float32)
    mask = np.ones((nz, ny, nx), np.uint8)
    vol = phantom.Volume(nx, ny, nz, S, 1, dy, f, mask)
    seeds = np.array([[nx / 2 + 0.5, ny / 2 + 0.5, nz / 2 + 0.5]], np.float32)
    return phantom.Workload("parity_box", vol, seeds, None, particles_per_seed=P, rng_seed=77)


def test_bidir_reverse_half_starts_against_d0():
    """R22: half 1 starts at the seed with previous direction -d0.  In the parity box its
    first draw (stream 1, block 0, word 0) is perpendicular to d0 iff the two sample
    indices differ in parity: then it ends CURV with 0 steps; otherwise its first step is
    exactly -d0.  d0 itself follows from stream 0, block 0 (sample word 0, sign word 3)."""
    w = _parity_box()
    S = w.volume.nsamples
    r = oracle.track(w.replace(bidir=1), path_stride=3)
    ns = r["nsteps"].reshape(-1, 2)
    why = r["reason"].reshape(-1, 2)
    paths = r["paths"].reshape(-1, 2, 3, 3)
    seed = w.seeds[0]
    curv = 0
    for i, pid in enumerate(_pids(w)):
        w0 = _words(w, pid, 0, 0)
        w1 = _words(w, pid, 0, 1)
        s0, s1 = (w0[0] * S) >> 32, (w1[0] * S) >> 32
        d0 = np.zeros(3, np.float32)
        d0[s0 % 2] = -1.0 if w0[3] >> 31 else 1.0
        assert np.array_equal(paths[i, 0, 1], seed + np.float32(0.5) * d0)
        if s0 % 2 != s1 % 2:
            curv += 1
            assert ns[i, 1] == 0 and why[i, 1] == oracle.END_CURV
            assert np.array_equal(r["end"].reshape(-1, 2, 3)[i, 1], seed)
        else:
            assert ns[i, 1] >= 1
            assert np.array_equal(paths[i, 1, 1], seed - np.float32(0.5) * d0)
    assert 0 < curv < len(ns)


def test_bidir_seed_outside_mask():
    """R12 + R22: both halves of a particle seeded outside the mask have 0 steps, MASK."""
    w = phantom.tube(particles_per_seed=5).replace(bidir=1)
    w = w.replace(seeds=np.array([[0.5, 0.5, 0.5], [-2.0, 3.0, 1.0]], np.float32))
    r = oracle.track(w)
    assert r["nsteps"].shape == (20,)
    assert np.all(r["nsteps"] == 0) and np.all(r["reason"] == oracle.END_MASK)
    assert np.array_equal(r["end"], np.repeat(w.seeds, 10, 0))


def test_bidir_connectivity_is_per_streamline():
    """NEXT-2 with R22: a streamline is the union of its halves, so in the tube every
    particle reaches both end slabs and counts once for each."""
    P = 30
    w = phantom.tube(particles_per_seed=P, seed_x=16)
    lab = np.zeros_like(w.volume.mask)
    lab[:, :, 24:26] = 1
    lab[:, :, 3:5] = 2
    one = oracle.track(w, labels=lab, ntargets=2)
    two = oracle.track(w.replace(bidir=1), labels=lab, ntargets=2)
    assert np.all(two["conn"] == P)
    assert np.array_equal(one["conn"].sum(1), np.full(w.nseeds, P))


# ----------------------------------------------------------------------------- R23 interpolation

def test_interp_bent_tube_per_particle():
    """R23 closed form: bent tube (x < 20: v = (1,0,0); x >= 20: v = (0,1,0)), seed at
    x = 8.5.  A forward particle at step n sits at x = 8.5 + n/2.  For even n the position
    is a voxel centre (weight 0: its own voxel); for odd n it lies half-way, so the voxel
    x+1 is sampled with probability 1/2.  It therefore reads the perpendicular fibre (CURV)
    first at n = 23 iff the x-uniform of stream 2, block 23 is < 1/2 (top bit 0), else at
    n = 24.  Backward particles never meet the bend: L- = 16, MASK (C-pin-5)."""
    w = phantom.bent_tube(0.0, particles_per_seed=400).replace(interp=1)
    r = oracle.track(w)
    sg = _signs(w)
    got23 = 0
    for i, pid in enumerate(_pids(w)):
        if sg[i] > 0:
            early = (_words(w, pid, 23, 2)[0] >> 31) == 0
            got23 += early
            assert r["nsteps"][i] == (23 if early else 24), i
            assert r["reason"][i] == oracle.END_CURV
        else:
            assert r["nsteps"][i] == 16 and r["reason"][i] == oracle.END_MASK
    fwd = int((sg > 0).sum())
    assert _binomial_ok(got23, fwd, 0.5)
    # without interpolation the nearest-voxel rule ends every forward particle at n = 23
    r0 = oracle.track(w.replace(interp=0))
    assert np.all(r0["nsteps"][sg > 0] == 23)


def test_interp_falls_back_to_the_nearest_voxel():
    """R23 fallback: seeds at y = 12.25 in the tube (mask y in [12, 20)): the y-neighbour
    below (voxel 11, outside the mask, weight 1/4) holds a perpendicular fibre with f = 1,
    so reading it would end the particle CURV.  With the fallback the lengths are exactly
    the tube's closed form (C-pin-5)."""
    w = phantom.tube(particles_per_seed=60, seed_x=16)
    v = w.volume
    dy = v.dyads.copy()
    f = v.f.copy()
    out = v.mask == 0
    dy[:, :, out] = np.array([0.0, 0.0, 1.0], np.float32)
    f[:, :, out] = 1.0
    vol = phantom.Volume(v.nx, v.ny, v.nz, v.nsamples, v.nfibres, dy, f, v.mask)
    seeds = np.array([[16.5, 12.25, 8.5]], np.float32)
    w = w.replace(volume=vol, seeds=seeds, interp=1)
    r = oracle.track(w)
    sg = _signs(w)
    assert np.array_equal(r["nsteps"], np.where(sg > 0, 30, 32))
    assert np.all(r["reason"] == oracle.END_MASK)
    # the fallback is exercised: about 1/4 of all steps' y-uniforms select voxel 11
    sel = tot = 0
    for pid, n in zip(_pids(w), r["nsteps"]):
        for k in range(int(n) + 1):
            tot += 1
            sel += (np.float32(_words(w, pid, k, 2)[1] >> 8) * np.float32(2.0 ** -24)) >= np.float32(0.75)
    assert _binomial_ok(sel, tot, 0.25)


def test_interp_voxel_frequencies_match_linear_weights():
    """R23 statistics: one step (max_steps = 1) from x = 7.5 + a, a in {1/8, 1/4, 3/8}.
    Voxels x >= 8 hold fibre (0,1,0), the others (1,0,0).  The sampled voxel is 8 with
    probability a (its linear weight), so a fraction a of the first steps go along y."""
    nx, ny, nz, S, P = 16, 8, 8, 4, 3000
    dy = np.zeros((1, S, nz, ny, nx, 3), np.float32)
    dy[..., 0] = 1.0
    dy[0, :, :, :, 8:, :] = np.array([0.0, 1.0, 0.0], np.float32)
    f = np.ones((1, S, nz, ny, nx), np.float32)
    mask = np.ones((nz, ny, nx), np.uint8)
    vol = phantom.Volume(nx, ny, nz, S, 1, dy, f, mask)
    for a in (0.125, 0.25, 0.375):
        seeds = np.array([[7.5 + a, 4.5, 4.5]], np.float32)
        w = phantom.Workload("interp_stat", vol, seeds, None, particles_per_seed=P,
                             max_steps=1, rng_seed=99, interp=1)
        r = oracle.track(w)
        moved_y = np.abs(r["end"][:, 1] - np.float32(4.5)) > 0
        assert _binomial_ok(int(moved_y.sum()), P, a), (a, int(moved_y.sum()))


# ----------------------------------------------------------------------------- R24 first fibre

def _fibre_box(fs, P=4000, mode=1, fib_thr=0.01):
    """F = len(fs); fibre j points along axis j everywhere with fraction fs[j]; one step."""
    F, S, nx, ny, nz = len(fs), 3, 12, 12, 12
    dy = np.zeros((F, S, nz, ny, nx, 3), np.float32)
    f = np.zeros((F, S, nz, ny, nx), np.float32)
    for j in range(F):
        dy[j, ..., j] = 1.0
        f[j] = np.float32(fs[j])
    mask = np.ones((nz, ny, nx), np.uint8)
    vol = phantom.Volume(nx, ny, nz, S, F, dy, f, mask)
    seeds = np.array([[6.5, 6.5, 6.5]], np.float32)
    w = phantom.Workload("fibre_box", vol, seeds, None, particles_per_seed=P, max_steps=1,
                         fib_thr=fib_thr, rng_seed=31, init_fibre=mode)
    r = oracle.track(w)
    axis = np.argmax(np.abs(r["end"] - seeds[0]), 1)
    assert np.all(r["nsteps"] == 1)
    return np.bincount(axis, minlength=3)


@pytest.mark.parametrize("fs,mode,probs", [
    ((0.5, 0.3), 0, (1.0, 0.0)),
    ((0.5, 0.3), 1, (0.5, 0.5)),
    ((0.5, 0.3), 2, (0.625, 0.375)),
    ((0.2, 0.0, 0.6), 1, (0.5, 0.0, 0.5)),
    ((0.2, 0.0, 0.6), 2, (0.25, 0.0, 0.75)),
    ((0.005, 0.4), 1, (0.0, 1.0)),
    ((0.005, 0.4), 0, (1.0, 0.0)),
    ((0.005, 0.008), 2, (1.0, 0.0)),
])
def test_first_fibre_frequencies(fs, mode, probs):
    """R24: first-step fibre frequencies: fibre 0 (mode 0, R5), uniform over the eligible
    fibres (mode 1), f-weighted over the eligible fibres (mode 2); no eligible fibre =>
    fibre 0; an ineligible fibre is never drawn."""
    counts = _fibre_box(fs, mode=mode)
    n = int(counts.sum())
    for j, p in enumerate(probs):
        if p in (0.0, 1.0):
            assert counts[j] == round(p * n), (j, counts)
        else:
            assert _binomial_ok(int(counts[j]), n, p), (j, counts)


# ----------------------------------------------------------------------------- brute force

@pytest.mark.parametrize("F,half,bidir,interp,init", [
    (1, False, 1, 0, 0), (2, False, 1, 1, 0), (2, True, 0, 1, 1), (3, False, 1, 1, 2),
    (3, True, 1, 0, 2), (2, False, 0, 0, 1),
])
def test_variants_bruteforce_bit_identical(F, half, bidir, interp, init):
    """C-pin-11 for the variants: every half's positions bit-identical to the numpy
    tracker, same nsteps and reasons; map = visits of all committed positions."""
    w = phantom.whole_brain(nx=14, ny=12, nz=10, semi=(6.0, 5.0, 4.0), nsamples=6, nfibres=F,
                            particles_per_seed=5, seeds="brain")
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 10))
    w = w.replace(curv_thr=0.3, bidir=bidir, interp=interp, init_fibre=init)
    if half:
        w = phantom.to_half(w)
    stride = 300
    r = oracle.track(w, path_stride=stride)
    H = 2 if bidir else 1
    m = np.zeros_like(r["map"])
    total = 0
    for i in range(w.nparticles):
        halves = bruteforce.track_streamline(w, i // w.particles_per_seed, i % w.particles_per_seed)
        assert len(halves) == H
        for h, (n, why, pos) in enumerate(halves):
            o = i * H + h
            assert (r["nsteps"][o], r["reason"][o]) == (n, why), (i, h)
            k = min(n + 1, stride)
            assert np.array_equal(r["paths"][o, :k].view(np.uint32), pos[:k].view(np.uint32)), (i, h)
            for x, y, z in pos[1:]:
                m[int(np.floor(z)), int(np.floor(y)), int(np.floor(x))] += 1
            total += n
    assert total > 2 * w.nparticles
    assert np.array_equal(r["map"], m)


def test_variant_invariants_and_arguments():
    """C-pin-10 with every variant on: sum(map) = sum over halves of nsteps, map = 0
    outside the mask, thread sharding and j-range splitting do not change anything;
    invalid variant values are rejected."""
    w = phantom.whole_brain(nx=24, ny=24, nz=16, semi=(10.0, 10.5, 6.5), nsamples=12,
                            particles_per_seed=24).replace(bidir=1, interp=1, init_fibre=2)
    r = oracle.track(w)
    assert int(r["map"].sum()) == int(r["nsteps"].sum())
    assert np.all(r["map"][w.volume.mask == 0] == 0)
    r3 = oracle.track(w, threads=3)
    for k in ("map", "nsteps", "reason", "end"):
        assert np.array_equal(r[k], r3[k])
    a = oracle.track(w, 0, 10)
    b = oracle.track(w, 10, 24)
    assert np.array_equal(a["map"] + b["map"], r["map"])
    for bad in (dict(bidir=2), dict(interp=-1), dict(init_fibre=3)):
        with pytest.raises(ValueError):
            oracle.track(w.replace(**bad))
