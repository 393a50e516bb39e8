"""Pins of the oracle against things other than itself (CPU only, ``-m "not gpu"``).

Each test names the pin of DESIGN.md "Parity and pins" it implements.  A plausible
mistake in oracle.c (dropped term, wrong sign or index, swapped operands, wrong tie
rule, wrong RNG word) must fail at least one of them.
"""
from __future__ import annotations

import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import phantom
from tests import bruteforce

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------------------- RNG (R16)

def _kat():
    rows = []
    for line in open(os.path.join(GOLDEN, "philox4x32_10_kat.txt")):
        if line.startswith("#") or not line.strip():
            continue
        v = [int(x, 16) for x in line.split()]
        rows.append((v[0:4], v[4:6], v[6:10]))
    return rows


@pytest.mark.parametrize("ctr,key,expect", _kat())
def test_philox_known_answers(ctr, key, expect):
    """C-pin-1: Random123 known-answer vectors (golden file, cited)."""
    assert list(oracle.philox(ctr, key)) == expect


def test_philox_matches_third_implementation():
    rng = np.random.default_rng(1)
    for _ in range(200):
        ctr = rng.integers(0, 2**32, 4, dtype=np.uint64)
        key = rng.integers(0, 2**32, 2, dtype=np.uint64)
        assert list(oracle.philox(ctr, key)) == bruteforce.philox4x32_10(ctr, key)


def test_sample_index_edges_and_buckets():
    """C-pin-2: s = floor(w S / 2^32): edge words and exact bucket boundaries."""
    for S in (1, 2, 3, 50, 4096, 65535):
        assert oracle.sample_index(0, S) == 0
        assert oracle.sample_index(2**32 - 1, S) == S - 1
        for s in list(range(1, min(S, 64))) + [S - 1]:
            if s <= 0:
                continue
            first = -(-(s << 32) // S)  # ceil(s 2^32 / S): first word of bucket s
            assert oracle.sample_index(first, S) == s
            assert oracle.sample_index(first - 1, S) == s - 1


def test_sample_index_uniform_chi2():
    """C-pin-2: the per-step sample draws are uniform over S (chi^2 over 10^5 draws)."""
    S = 50
    counts = np.zeros(S, np.int64)
    key = (0x1234, 0x5678)
    n = 0
    for pid in range(25000):
        w = oracle.philox([0, pid, 0, 0], key)
        for word in w[:3]:
            counts[oracle.sample_index(int(word), S)] += 1
            n += 1
    e = n / S
    chi2 = ((counts - e) ** 2 / e).sum()
    # 49 dof: P(chi2 > 85) ~ 1e-3
    assert chi2 < 85, chi2


def test_init_sign_is_fair():
    key = (7, 9)
    ones = sum(int(oracle.philox([0, pid, 0, 0], key)[3]) >> 31 for pid in range(20000))
    assert abs(ones - 10000) < 4 * math.sqrt(5000)


# ----------------------------------------------------------------------------- fp16 (R15)

def test_half_decode_exhaustive():
    """C-pin-3: all 65536 binary16 patterns vs numpy's float16 -> float32 cast."""
    bits = np.arange(65536, dtype=np.uint32).astype(np.uint16)
    got = oracle.half_to_float(bits)
    ref = bits.view(np.float16).astype(np.float32)
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(got[~nan].view(np.uint32), ref[~nan].view(np.uint32))


# ----------------------------------------------------------------------------- lookup (R10)

def _r10(q: float, n: int) -> int:
    """R10 stated with exact rationals: c + floor(q) for q >= +0, c - floor(|q|) - 1 for
    q <= -0 (so exact integer boundaries resolve away from the volume centre)."""
    c = n // 2
    fq = Fraction(q)
    if fq > 0 or (fq == 0 and math.copysign(1.0, q) > 0):
        return c + math.floor(fq)
    return c - math.floor(-fq) - 1


def test_axis_index_boundaries():
    """C-pin-4: +-0, +-0.5, +-k, +-(k - 1 ulp)."""
    n = 32
    c = 16
    assert oracle.axis_index(0.0, n) == c
    assert oracle.axis_index(-0.0, n) == c - 1
    assert oracle.axis_index(0.5, n) == c
    assert oracle.axis_index(-0.5, n) == c - 1
    for k in range(1, 6):
        assert oracle.axis_index(float(k), n) == c + k
        assert oracle.axis_index(float(-k), n) == c - k - 1
        below = float(np.nextafter(np.float32(k), np.float32(0)))
        assert oracle.axis_index(below, n) == c + k - 1
        assert oracle.axis_index(-below, n) == c - k
    rng = np.random.default_rng(3)
    for q in rng.uniform(-20, 20, 2000).astype(np.float32):
        assert oracle.axis_index(float(q), n) == _r10(float(q), n)
        # mirror: voxel(-q) = N - 1 - voxel(q) for even N, q != 0
        assert oracle.axis_index(float(-q), n) == n - 1 - oracle.axis_index(float(q), n)
    assert oracle.axis_index(float(33), 33) == 33 // 2 + 33


# ----------------------------------------------------------------------------- closed forms

def _exact_path(N, xs, sign, n):
    """Exact corner x-coordinates and voxels of a particle stepping 0.5 along +-x."""
    c = N // 2
    q0 = Fraction(2 * xs + 1, 2) - c
    out = []
    for k in range(1, n + 1):
        q = q0 + sign * Fraction(k, 2)
        # an exact zero reached by stepping is +0 in IEEE RNE (x + (-x) = +0)
        out.append(c + math.floor(q) if q >= 0 else c - math.floor(-q) - 1)
    return out


def _signs(w):
    key = (w.rng_seed & 0xFFFFFFFF, w.rng_seed >> 32)
    P = w.particles_per_seed
    out = []
    for sid in w.ids():
        for j in range(P):
            pid = int(sid) * P + j
            out.append(-1 if int(oracle.philox([0, pid & 0xFFFFFFFF, pid >> 32, 0], key)[3]) >> 31 else 1)
    return np.array(out)


def _tube_rows():
    rows = []
    for line in open(os.path.join(GOLDEN, "tube_closed_form.txt")):
        if line.startswith("#") or not line.strip():
            continue
        rows.append(tuple(int(x) for x in line.split()))
    return rows


@pytest.mark.parametrize("N,x0,x1,xs,Lp,Lm", _tube_rows())
def test_straight_tube_closed_form(N, x0, x1, xs, Lp, Lm):
    """C-pin-5: zero-dispersion tube: lengths, reason, end points and map exactly."""
    w = phantom.tube(nx=N, x=(x0, x1 + 1), seed_x=xs, particles_per_seed=40)
    r = oracle.track(w)
    sg = _signs(w)
    L = np.where(sg > 0, Lp, Lm)
    assert np.array_equal(r["nsteps"], L)
    assert np.all(r["reason"] == oracle.END_MASK)
    ex = (np.float32(xs) + np.float32(0.5) + np.float32(0.5) * sg * L).astype(np.float32)
    assert np.array_equal(r["end"][:, 0], ex)
    seeds = np.repeat(w.seeds, w.particles_per_seed, 0)
    assert np.array_equal(r["end"][:, 1:], seeds[:, 1:])
    # map: every committed step's voxel from the exact rational path
    m = np.zeros_like(r["map"])
    for i, (s, n) in enumerate(zip(sg, L)):
        sy, sz = seeds[i, 1].astype(int), seeds[i, 2].astype(int)
        for vx in _exact_path(N, xs, s, int(n)):
            m[sz, sy, vx] += 1
    assert np.array_equal(r["map"], m)


def test_straight_tube_max_steps():
    """C-pin-5 with max_steps = m: L = min(L+-, m), MAXLEN iff L+- >= m."""
    w = phantom.tube(particles_per_seed=30, max_steps=31)
    r = oracle.track(w)
    sg = _signs(w)
    full = np.where(sg > 0, 30, 32)
    assert np.array_equal(r["nsteps"], np.minimum(full, 31))
    assert np.array_equal(r["reason"], np.where(full >= 31, oracle.END_MAXLEN, oracle.END_MASK))


def test_c1_config_counts():
    """c1 (BASELINE configs[0]) as generated: c = 16, xs = 16, full tube: 30 / 32."""
    w = phantom.config("c1")
    r = oracle.track(w)
    sg = _signs(w)
    assert np.array_equal(r["nsteps"], np.where(sg > 0, 30, 32))
    assert int(r["map"].sum()) == int(r["nsteps"].sum())


def test_t_junction_terminates_on_curvature():
    """C-pin-7: bundle A ends in a B-only column at x_J: the particle commits the step
    into voxel x_J and ends CURV there (|dot| = 0 <= curv_thr); backwards it runs to x=0."""
    xJ = 40
    w = phantom.t_junction(x_j=xJ, seed_xs=(20, 30), particles_per_seed=100)
    r = oracle.track(w)
    sg = _signs(w)
    N = w.volume.nx
    for i in range(w.nparticles):
        xs = int(w.seeds[i // w.particles_per_seed][0])
        if sg[i] > 0:
            vox = _exact_path(N, xs, 1, 200)
            k = vox.index(xJ) + 1          # first step landing in the junction column
            assert r["nsteps"][i] == k and r["reason"][i] == oracle.END_CURV
            assert int(math.floor(r["end"][i][0])) == xJ
        else:
            vox = _exact_path(N, xs, -1, 200)
            k = vox.index(-1)              # steps until leaving the volume at x < 0
            assert r["nsteps"][i] == k and r["reason"][i] == oracle.END_MASK


@pytest.mark.parametrize("at_threshold", [True, False])
def test_bent_tube_threshold_tie(at_threshold):
    """C-pin-6: v2 = (c, s, 0) with fp32 dot exactly c: ends CURV iff not c > curv_thr."""
    thr = np.float32(0.2)
    cval = thr if at_threshold else np.nextafter(thr, np.float32(1))
    xb = 20
    w = phantom.bent_tube(float(cval), x_bend=xb, curv_thr=float(thr), particles_per_seed=64)
    r = oracle.track(w)
    sg = _signs(w)
    xs = int(w.seeds[0][0])
    kb = _exact_path(w.volume.nx, xs, 1, 100).index(xb) + 1   # first step into the bend
    fwd = sg > 0
    if at_threshold:
        assert np.all(r["nsteps"][fwd] == kb)
        assert np.all(r["reason"][fwd] == oracle.END_CURV)
    else:
        assert np.all(r["nsteps"][fwd] > kb)
        assert np.all(r["reason"][fwd] == oracle.END_MASK)
    assert np.all(r["reason"][~fwd] == oracle.END_MASK)
    assert np.all(r["nsteps"][~fwd] == _exact_path(w.volume.nx, xs, -1, 100).index(-1))


def test_crossing_keeps_bundle():
    """C-pin-7: 90 degree crossing, zero dispersion: a particle keeps its bundle through
    the crossing (the perpendicular fibre has |dot| = 0), so lengths are the tube's."""
    w = phantom.crossing(nseeds=60, particles_per_seed=20)
    r = oracle.track(w)
    sg = _signs(w)
    N = 64
    A_y = (24, 40)
    for i in range(w.nparticles):
        x, y, z = (int(t) for t in w.seeds[i // w.particles_per_seed])
        along_x = A_y[0] <= y < A_y[1]        # bundle A (or the crossing: fibre 0 = A)
        xs = x if along_x else y
        path = _exact_path(N, xs, int(sg[i]), 200)
        k = path.index(-1) if sg[i] < 0 else path.index(N)
        assert r["nsteps"][i] == k, (i, x, y, z)
        assert r["reason"][i] == oracle.END_MASK
        e = r["end"][i]
        if along_x:
            assert e[1] == y + 0.5 and e[2] == z + 0.5
        else:
            assert e[0] == x + 0.5 and e[2] == z + 0.5


# ----------------------------------------------------------------------------- symmetry

def test_mirror_symmetry_dispersed():
    """C-pin-8: mirrored dispersed crossing phantom with the same seed ids: maps mirror
    bit-exactly, (nsteps, reason) equal per pid, end points mirror in x."""
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=40, particles_per_seed=50, nsamples=20)
    m = phantom.mirror_x(w)
    a = oracle.track(w)
    b = oracle.track(m)
    assert np.array_equal(a["nsteps"], b["nsteps"])
    assert np.array_equal(a["reason"], b["reason"])
    assert np.array_equal(a["map"][:, :, ::-1], b["map"])
    assert np.allclose(a["end"][:, 0] + b["end"][:, 0], 64.0, atol=1e-5)
    assert np.array_equal(a["end"][:, 1:], b["end"][:, 1:])
    assert a["nsteps"].sum() > 10 * w.nparticles


# ----------------------------------------------------------------------------- statistics

@pytest.mark.parametrize("F,thr", [(1, 0.2), (2, 0.2), (2, 0.5)])
def test_isotropic_geometric_law(F, thr):
    """C-pin-9 (and Eq. 4): with isotropic samples the curvature hazard per
    step is thr^F (|u.d| ~ U[0,1], Archimedes), so n ~ Geometric(p = thr^F) on {1,2,..}:
    the exponential fibre-length law of P:L245 in discrete form."""
    w = phantom.isotropic(n=24, nsamples=512, nfibres=F, nseeds=4, particles_per_seed=5000,
                          curv_thr=thr)
    r = oracle.track(w)
    n = r["nsteps"]
    curv = r["reason"] == oracle.END_CURV
    p = thr ** F
    # hazard estimate with exits as censoring: every particle with n >= 1 performed
    # exactly n curvature tests (iterations at n = 1..n); the CURV-ended ones failed one.
    tests = int(n.sum())
    ph = curv.sum() / tests
    assert abs(ph - p) < 4 * math.sqrt(p * (1 - p) / tests), (ph, p)
    # distribution of the uncensored lengths: Geometric(p) on {1, 2, ...}
    if curv.mean() > 0.995:
        n = n[curv]
        K = max(3, int(3 / p))
        obs = np.array([(n == k).sum() for k in range(1, K + 1)] + [(n > K).sum()], float)
        pk = np.array([(1 - p) ** (k - 1) * p for k in range(1, K + 1)] + [(1 - p) ** K])
        e = pk * n.size
        chi2 = ((obs - e) ** 2 / e).sum()
        assert chi2 < K + 1 + 6 * math.sqrt(2 * (K + 1)), (chi2, K)


# ----------------------------------------------------------------------------- invariants

def _small_brain(F=2, P=40):
    return phantom.whole_brain(nx=24, ny=24, nz=16, semi=(10.0, 10.5, 6.5), nsamples=12,
                               nfibres=F, particles_per_seed=P)


def test_global_invariants():
    """C-pin-10: sum(map) = sum(nsteps); map = 0 outside the mask; nsteps <= max_steps;
    j-range splitting, thread sharding and seed-order permutation invariance."""
    w = _small_brain()
    r = oracle.track(w)
    assert int(r["map"].sum()) == int(r["nsteps"].sum())
    assert np.all(r["map"][w.volume.mask == 0] == 0)
    assert r["nsteps"].max() <= w.max_steps
    r2 = oracle.track(w, threads=3)
    for k in ("map", "nsteps", "reason", "end"):
        assert np.array_equal(r[k], r2[k])
    a = oracle.track(w, 0, 17)
    b = oracle.track(w, 17, 40)
    assert np.array_equal(a["map"] + b["map"], r["map"])
    ns = r["nsteps"].reshape(w.nseeds, 40)
    assert np.array_equal(np.concatenate([a["nsteps"].reshape(-1, 17), b["nsteps"].reshape(-1, 23)], 1), ns)
    perm = np.random.default_rng(0).permutation(w.nseeds)
    wp = w.replace(seeds=w.seeds[perm].copy(), seed_ids=w.ids()[perm].copy())
    rp = oracle.track(wp)
    assert np.array_equal(rp["map"], r["map"])
    assert np.array_equal(rp["nsteps"].reshape(w.nseeds, 40), ns[perm])


def test_seed_outside_mask_and_argument_checks():
    """R12: a seed outside the mask gives 0 steps, reason MASK, end = seed."""
    w = _small_brain(P=3)
    w = w.replace(seeds=np.array([[0.5, 0.5, 0.5], [-3.0, 2.0, 1.0]], np.float32))
    r = oracle.track(w)
    assert np.all(r["nsteps"] == 0) and np.all(r["reason"] == oracle.END_MASK)
    assert np.array_equal(r["end"], np.repeat(w.seeds, 3, 0))
    with pytest.raises(ValueError):
        oracle.track(w.replace(max_steps=0))
    with pytest.raises(ValueError):
        oracle.track(w.replace(step=-1.0))
    with pytest.raises(ValueError):
        oracle.track(w.replace(curv_thr=1.5))


# ----------------------------------------------------------------------------- brute force

@pytest.mark.parametrize("half", [False, True])
@pytest.mark.parametrize("F", [1, 2, 3])
def test_bruteforce_paths_bit_identical(F, half):
    """C-pin-11: numpy-float32 third implementation on a tiny volume: every position of
    every path bit-identical, same nsteps and reason."""
    w = phantom.whole_brain(nx=14, ny=12, nz=10, semi=(6.0, 5.0, 4.0), nsamples=6, nfibres=F,
                            particles_per_seed=6, seeds="brain")
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 12))
    w = w.replace(curv_thr=0.3)
    if half:
        w = phantom.to_half(w)
    stride = 400
    r = oracle.track(w, path_stride=stride)
    total = 0
    for i in range(w.nparticles):
        n, why, pos = bruteforce.track(w, i // w.particles_per_seed, i % w.particles_per_seed)
        assert (r["nsteps"][i], r["reason"][i]) == (n, why), i
        k = min(n + 1, stride)
        assert np.array_equal(r["paths"][i, :k].view(np.uint32), pos[:k].view(np.uint32)), i
        total += n
    assert total > 3 * w.nparticles


# ----------------------------------------------------------------------------- fibre choice

def _fork_ends(after, **kw):
    w = phantom.fork(after, **kw)
    r = oracle.track(w)
    fwd = _signs(w) > 0
    return w, r, fwd


def test_fibre_tie_lowest_index_wins():
    """R8: two fibres with exactly equal |dot| (fp32 dot = c for both): the lower index
    wins, so forward particles turn to +y (fibre 0 = (c, s, 0), fibre 1 = (c, -s, 0))."""
    c = np.float32(0.6)
    s = np.float32(math.sqrt(1 - float(c) ** 2))
    w, r, fwd = _fork_ends([((c, s, 0), 0.5), ((c, -s, 0), 0.5)])
    y0 = w.seeds[0][1]
    assert np.all(r["end"][fwd, 1] > y0 + 2)
    assert np.all(r["end"][~fwd, 1] == y0)
    # swapped order: fibre 0 now points to -y
    w, r, fwd = _fork_ends([((c, -s, 0), 0.5), ((c, s, 0), 0.5)])
    assert np.all(r["end"][fwd, 1] < y0 - 2)
    # equal |dot| with opposite signs: fibre 0 = (-c, s, 0) wins and is flipped (R9)
    w, r, fwd = _fork_ends([((-c, s, 0), 0.5), ((c, -s, 0), 0.5)])
    assert np.all(r["end"][fwd, 1] < y0 - 2) and np.all(r["end"][fwd, 0] > 20)


def test_fibre_eligibility_is_strict():
    """R7: a fibre with f == fib_thr exactly is not eligible; the eligible fibre 1 wins
    although fibre 0 is better aligned."""
    c = np.float32(0.6)
    s = np.float32(math.sqrt(1 - float(c) ** 2))
    thr = np.float32(0.01)
    w, r, fwd = _fork_ends([((1, 0, 0), thr), ((c, -s, 0), 0.5)], fib_thr=float(thr))
    y0 = w.seeds[0][1]
    assert np.all(r["end"][fwd, 1] < y0 - 2)
    w, r, fwd = _fork_ends([((1, 0, 0), np.nextafter(thr, np.float32(1))), ((c, -s, 0), 0.5)],
                           fib_thr=float(thr))
    assert np.all(r["end"][fwd, 1] == y0)


def test_no_eligible_fibre_continues_on_fibre0():
    """R7: no eligible fibre => fibre 0, never a termination on f."""
    w, r, fwd = _fork_ends([((1, 0, 0), 0.0), ((0, 1, 0), 0.0)])
    xs = int(w.seeds[0][0])
    assert np.all(r["nsteps"][fwd] == _exact_path(w.volume.nx, xs, 1, 200).index(w.volume.nx))
    assert np.all(r["reason"] == oracle.END_MASK)


def test_zero_dot_sign_is_negative():
    """R9: with curv_thr < 0 a zero dot passes the angle test and the sign is -1: at the
    T-junction (fibre (0,1,0), previous direction (1,0,0), dot = +0) forward particles
    turn to -y and run to the y = 0 face."""
    w = phantom.t_junction(x_j=40, seed_xs=(30,), particles_per_seed=64, curv_thr=-0.5)
    r = oracle.track(w)
    fwd = _signs(w) > 0
    assert np.all(r["reason"] == oracle.END_MASK)
    assert np.all(r["end"][fwd, 1] < 1.0)
    assert np.all(r["end"][fwd, 0] >= 40)


# ----------------------------------------------------------------------------- NEXT-1 paper mode

def _alternating_tube(nx=40, ny=40, nz=8, S=4, P=24, seed_xy=(20, 20)):
    """Whole-volume mask; sample s points along x for even s, along y for odd s (F = 1)."""
    dy = np.zeros((1, S, nz, ny, nx, 3), np.float32)
    for s in range(S):
        dy[0, s, ..., 0 if s % 2 == 0 else 1] = 1.0
    f = np.ones((1, S, nz, ny, nx), np.float32)
    mask = np.ones((nz, ny, nx), np.uint8)
    vol = phantom.Volume(nx, ny, nz, S, 1, dy, f, mask)
    seeds = np.array([[seed_xy[0] + 0.5, seed_xy[1] + 0.5, nz // 2 + 0.5]], np.float32)
    return phantom.Workload("alt_tube", vol, seeds, None, particles_per_seed=P, rng_seed=99,
                            sample_mode=1)


def test_paper_mode_one_sample_per_streamline():
    """NEXT-1 (Alg. 1: each streamline follows one sample volume):
    particle j uses sample j mod S for every step, so with samples alternating between
    +-x and +-y it runs straight along x (j even) or y (j odd) to the volume face."""
    w = _alternating_tube()
    r = oracle.track(w)
    sg = _signs(w)
    N = 40
    for j in range(w.particles_per_seed):
        path = _exact_path(N, 20, int(sg[j]), 200)
        k = path.index(-1) if sg[j] < 0 else path.index(N)
        assert r["nsteps"][j] == k and r["reason"][j] == oracle.END_MASK
        e = r["end"][j]
        moved, fixed = (0, 1) if j % 2 == 0 else (1, 0)
        assert e[fixed] == 20.5
        assert e[moved] == np.float32(20.5 + 0.5 * sg[j] * k)
    # the per-step random mode (R1) mixes the two directions instead
    rr = oracle.track(w.replace(sample_mode=0))
    assert not np.array_equal(rr["nsteps"], r["nsteps"])


@pytest.mark.parametrize("half", [False, True])
def test_paper_mode_bruteforce(half):
    w = phantom.whole_brain(nx=14, ny=12, nz=10, semi=(6.0, 5.0, 4.0), nsamples=6, nfibres=2,
                            particles_per_seed=6, seeds="brain")
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 12)).replace(curv_thr=0.3, sample_mode=1)
    if half:
        w = phantom.to_half(w)
    r = oracle.track(w, path_stride=300)
    for i in range(w.nparticles):
        n, why, pos = bruteforce.track(w, i // w.particles_per_seed, i % w.particles_per_seed)
        assert (r["nsteps"][i], r["reason"][i]) == (n, why), i
        k = min(n + 1, 300)
        assert np.array_equal(r["paths"][i, :k].view(np.uint32), pos[:k].view(np.uint32)), i
    with pytest.raises(ValueError):
        oracle.track(w.replace(sample_mode=2))


# ----------------------------------------------------------------------------- NEXT-2 connectivity

def test_connectivity_tube_closed_form():
    """NEXT-2 (count the streamlines passing through B): tube with two target slabs.
    A particle counts once for a target iff its exact rational path (committed steps, R21)
    enters a voxel of the slab, however many steps it spends there."""
    w = phantom.tube(particles_per_seed=50, seed_x=16)
    nx = w.volume.nx
    lab = np.zeros_like(w.volume.mask)
    lab[:, :, 24:26] = 1      # ahead in +x
    lab[:, :, 3:5] = 2        # behind
    lab[:, :, 16] = 3         # the seed voxel column
    r = oracle.track(w, labels=lab, ntargets=3)
    sg = _signs(w)
    expect = np.zeros((w.nseeds, 3), np.uint64)
    for i in range(w.nparticles):
        s = i // w.particles_per_seed
        path = _exact_path(nx, 16, int(sg[i]), int(r["nsteps"][i]))
        hit = {1: any(24 <= v <= 25 for v in path), 2: any(3 <= v <= 4 for v in path),
               3: any(v == 16 for v in path)}
        for t in (1, 2, 3):
            expect[s, t - 1] += hit[t]
    assert np.array_equal(r["conn"], expect)
    # every forward particle passes target 1, every backward one target 2; target 3 (the
    # seed voxel) is entered again only by backward particles (q = +0 lands in voxel c)
    fwd = (sg > 0).reshape(w.nseeds, -1).sum(1)
    assert np.array_equal(r["conn"][:, 0], fwd) and np.array_equal(r["conn"][:, 1], 50 - fwd)
    assert np.array_equal(r["conn"][:, 2], 50 - fwd)


def test_connectivity_matches_bruteforce_paths():
    """NEXT-2 on a dispersed brain: the oracle's matrix equals one computed from the numpy
    brute-force tracker's positions and the label volume."""
    w = phantom.whole_brain(nx=16, ny=14, nz=10, semi=(7.0, 6.0, 4.0), nsamples=6, nfibres=2,
                            particles_per_seed=8, seeds="brain")
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 10)).replace(curv_thr=0.3)
    rng = np.random.default_rng(4)
    lab = (rng.integers(0, 5, w.volume.mask.shape) * (rng.random(w.volume.mask.shape) < 0.3)).astype(np.uint8)
    r = oracle.track(w, labels=lab, ntargets=4)
    expect = np.zeros((w.nseeds, 4), np.uint64)
    for i in range(w.nparticles):
        n, why, pos = bruteforce.track(w, i // w.particles_per_seed, i % w.particles_per_seed)
        got = set()
        for x, y, z in pos[1:]:  # committed positions (R21)
            vx = int(np.floor(x)); vy = int(np.floor(y)); vz = int(np.floor(z))
            if lab[vz, vy, vx]:
                got.add(int(lab[vz, vy, vx]))
        for t in got:
            expect[i // w.particles_per_seed, t - 1] += 1
    assert np.array_equal(r["conn"], expect)
    assert r["conn"].sum() > 0
