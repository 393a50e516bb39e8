"""Pins of the NEXT-2 per-streamline-unique visitation map in the oracle (R25; P:L109
"counting the number of streamlines passing through B, and dividing it by the total number
of the streamlines").  CPU only.

umap[v] = number of streamlines with at least one committed step landing in voxel v (the
seed position itself is not a visit, as in R13 / R21; a bidirectional streamline is the
union of its two halves).  Pinned by: the straight-tube closed form (the exact rational
path's voxel set), a numpy brute-force tracker's voxel sets, and invariants that a dropped
or double count would break (umap <= map, umap <= streamlines, closed loops where the two
maps differ)."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import phantom
from tests import bruteforce
from tests.test_oracle_pins import _exact_path, _signs


def test_unique_tube_closed_form():
    """Straight tube (C-pin-5 geometry): every particle enters each voxel of its exact
    rational path once, so umap is the sum of the path voxel SETS, while map sums the path
    voxel LISTS (a voxel holds two 0.5 steps)."""
    w = phantom.tube(particles_per_seed=40, seed_x=16)
    r = oracle.track(w, want_unique=True)
    sg = _signs(w)
    seeds = np.repeat(w.seeds, w.particles_per_seed, 0)
    u = np.zeros_like(r["umap"])
    for i, (s, n) in enumerate(zip(sg, r["nsteps"])):
        sy, sz = int(seeds[i, 1]), int(seeds[i, 2])
        for vx in set(_exact_path(w.volume.nx, 16, int(s), int(n))):
            u[sz, sy, vx] += 1
    assert np.array_equal(r["umap"], u)
    assert r["umap"].sum() < r["map"].sum()
    assert r["umap"].max() <= w.nparticles


@pytest.mark.parametrize("bidir", [0, 1])
@pytest.mark.parametrize("sigma", [0.0, 0.2])
def test_unique_matches_bruteforce_voxel_sets(bidir, sigma):
    """Closed loops (vortex annulus, ~3 turns per streamline): umap equals the histogram of
    the brute-force tracker's per-streamline voxel sets, union of both halves with bidir."""
    w = phantom.vortex(sigma=sigma, particles_per_seed=6, max_steps=500, nseeds_per_r=2).replace(bidir=bidir)
    r = oracle.track(w, want_unique=True)
    expect = np.zeros_like(r["umap"])
    for si in range(w.nseeds):
        for j in range(w.particles_per_seed):
            for (z, y, x) in bruteforce.streamline_voxels(w, si, j):
                expect[z, y, x] += 1
    assert np.array_equal(r["umap"], expect)
    # loops: the step map counts revisits, the unique map does not
    assert r["map"].sum() > 1.5 * r["umap"].sum()
    assert np.all(r["umap"] <= r["map"])
    assert r["umap"].max() <= w.nparticles


def test_unique_brain_bruteforce_and_invariants():
    """Dispersed brain-shaped volume, F = 3: umap from the brute-force voxel sets; umap = 0
    outside the mask; umap <= map; summing per-seed-shard umaps gives the full umap."""
    w = phantom.whole_brain(nx=16, ny=14, nz=10, semi=(7.0, 6.0, 4.0), nsamples=6, nfibres=3,
                            particles_per_seed=8, seeds="brain")
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 12)).replace(curv_thr=0.1)
    r = oracle.track(w, want_unique=True)
    expect = np.zeros_like(r["umap"])
    for si in range(w.nseeds):
        for j in range(w.particles_per_seed):
            for (z, y, x) in bruteforce.streamline_voxels(w, si, j):
                expect[z, y, x] += 1
    assert np.array_equal(r["umap"], expect)
    assert np.all(r["umap"][w.volume.mask == 0] == 0)
    assert np.all(r["umap"] <= r["map"])
    half = [phantom.wm_seeds(w.replace(seeds=w.seeds[k::2].copy(), seed_ids=w.ids()[k::2].copy()), 1)
            for k in (0, 1)]
    tot = sum(oracle.track(h, want_unique=True)["umap"] for h in half)
    assert np.array_equal(tot, r["umap"])


def test_unique_equals_map_without_revisits():
    """A particle that never returns to a voxel: straight tube at step 1.0 (one step per
    voxel), so every committed step enters a new voxel and umap == map exactly."""
    w = phantom.tube(particles_per_seed=20, seed_x=16).replace(step=1.0)
    r = oracle.track(w, want_unique=True)
    assert np.array_equal(r["umap"], r["map"])
    assert r["umap"].sum() == r["nsteps"].sum()
