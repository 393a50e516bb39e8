"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This module only *generates data*: per-voxel ball-and-stick orientation samples (the
six sample volumes of P:L125 / Fig. 1, already converted from (theta, phi) to
Cartesian unit vectors), a tracking mask and seed points.  It contains
none of the tracking arithmetic: no stepping, no RNG contract, no voxel lookup.  Both
``oracle/`` and the CUDA binding consume the arrays it returns; neither is imported here.

Canonical layout (the C-ABI's and the oracle's input format):

* ``dyads`` : ``[F][S][Z][Y][X][3]`` float32 (or float16), x fastest, xyz innermost
* ``f``     : ``[F][S][Z][Y][X]``   float32 (or float16)
* ``mask``  : ``[Z][Y][X]``         uint8, != 0 inside
* ``seeds`` : ``[nseeds][3]``       float32 corner-convention voxel coordinates
  (x, y, z); the centre of voxel i is i + 0.5.

Every generator is driven by ``numpy.random.Generator(PCG64(seed))``; the recipe of
each configuration is stated in DESIGN.md ("Input recipe") and mirrors the shapes of
BASELINE.json ``configs`` (c1..c5).
"""
from __future__ import annotations

import dataclasses
import hashlib
import math
from typing import Optional

import numpy as np

__all__ = [
    "Volume", "Workload", "tube", "crossing", "whole_brain", "isotropic", "bent_tube",
    "t_junction", "fork", "vortex", "paper_dataset", "mirror_x", "to_half", "config", "CONFIGS", "wm_seeds",
    "DwiWorkload", "gradient_scheme", "dwi_brain", "dwi_uniform", "MCMC_CONFIGS", "mcmc_config",
]


@dataclasses.dataclass
class Volume:
    nx: int
    ny: int
    nz: int
    nsamples: int
    nfibres: int
    dyads: np.ndarray  # [F][S][Z][Y][X][3]
    f: np.ndarray      # [F][S][Z][Y][X]
    mask: np.ndarray   # [Z][Y][X] uint8

    @property
    def is_half(self) -> bool:
        return self.dyads.dtype == np.float16

    @property
    def dtype(self) -> str:
        return "f16" if self.is_half else "f32"

    def sha256(self) -> str:
        h = hashlib.sha256()
        for a in (self.dyads, self.f, self.mask):
            h.update(np.ascontiguousarray(a).tobytes())
        return h.hexdigest()

    def check(self) -> None:
        F, S, Z, Y, X = self.nfibres, self.nsamples, self.nz, self.ny, self.nx
        assert self.dyads.shape == (F, S, Z, Y, X, 3), self.dyads.shape
        assert self.f.shape == (F, S, Z, Y, X), self.f.shape
        assert self.mask.shape == (Z, Y, X) and self.mask.dtype == np.uint8
        assert self.dyads.dtype == self.f.dtype
        assert self.dyads.flags.c_contiguous and self.f.flags.c_contiguous


@dataclasses.dataclass
class Workload:
    name: str
    volume: Volume
    seeds: np.ndarray                 # [nseeds][3] float32 corner coords
    seed_ids: Optional[np.ndarray]    # [nseeds] uint64 or None (=> 0..nseeds-1)
    step: float = 0.5
    curv_thr: float = 0.2
    fib_thr: float = 0.01
    max_steps: int = 2000
    rng_seed: int = 0x5EED_2012
    particles_per_seed: int = 1000
    recipe: str = ""
    sample_mode: int = 0  # 0: random sample per step (R1); 1: paper mode, s = j mod S (NEXT-1)
    # NEXT-3 FSL-fidelity variants (R22-R24)
    bidir: int = 0        # 1: bidirectional streamlines (two halves per particle)
    interp: int = 0       # 1: probabilistic interpolation of the sampled voxel
    init_fibre: int = 0   # first-step fibre: 0 fibre 0, 1 uniform eligible, 2 f-weighted

    @property
    def nseeds(self) -> int:
        return int(self.seeds.shape[0])

    @property
    def nparticles(self) -> int:
        return self.nseeds * self.particles_per_seed

    def ids(self) -> np.ndarray:
        if self.seed_ids is None:
            return np.arange(self.nseeds, dtype=np.uint64)
        return self.seed_ids

    def replace(self, **kw) -> "Workload":
        return dataclasses.replace(self, **kw)


# ----------------------------------------------------------------------------- helpers

def _normalize(v: np.ndarray) -> np.ndarray:
    n = np.sqrt((v.astype(np.float64) ** 2).sum(-1, keepdims=True))
    n[n == 0] = 1.0
    return (v / n).astype(np.float32)


def _centres(idx: np.ndarray) -> np.ndarray:
    """Voxel-centre corner coordinates (i + 0.5) for integer indices [n][3] (x,y,z)."""
    return np.ascontiguousarray((idx.astype(np.float32) + np.float32(0.5)).astype(np.float32))


def _empty(nx, ny, nz, S, F):
    dy = np.zeros((F, S, nz, ny, nx, 3), np.float32)
    dy[..., 0] = 1.0
    f = np.zeros((F, S, nz, ny, nx), np.float32)
    mask = np.zeros((nz, ny, nx), np.uint8)
    return dy, f, mask


def _disperse(v: np.ndarray, sigma, rng: np.random.Generator) -> np.ndarray:
    """normalize(v + sigma * N(0, I3)) in float32: a Watson/vMF-like per-sample spread.

    sigma = 0.15 gives ~10-12 degrees mean angular deviation (SURVEY §8(d) c2 recipe).
    """
    g = rng.standard_normal(v.shape, dtype=np.float32)
    if np.ndim(sigma):
        sigma = np.asarray(sigma, np.float32)[..., None]
    return _normalize(v + np.float32(1) * sigma * g)


# ----------------------------------------------------------------------------- c1

def tube(nx=32, ny=32, nz=16, y=(12, 20), z=(4, 12), x=(0, 32), nsamples=50,
         seed_x=16, particles_per_seed=1000, step=0.5, max_steps=2000, curv_thr=0.2,
         rng_seed=0x5EED_2012, direction=(1.0, 0.0, 0.0)) -> Workload:
    """c1: zero-dispersion straight tube along x (BASELINE.json configs[0]).

    Mask = the tube x in [x0,x1), y in [y0,y1), z in [z0,z1); F = 1; every sample is
    ``direction`` with f = 1.  Seeds: the 8x8 cross-section voxel centres at x = seed_x.
    """
    F, S = 1, nsamples
    dy, f, mask = _empty(nx, ny, nz, S, F)
    mask[z[0]:z[1], y[0]:y[1], x[0]:x[1]] = 1
    dy[...] = np.asarray(direction, np.float32)
    f[:, :, z[0]:z[1], y[0]:y[1], x[0]:x[1]] = 1.0
    vol = Volume(nx, ny, nz, S, F, dy, f, mask)
    yy, zz = np.meshgrid(np.arange(*y), np.arange(*z), indexing="xy")
    idx = np.stack([np.full(yy.size, seed_x), yy.ravel(), zz.ravel()], 1)
    seeds = _centres(idx)
    return Workload("c1_tube", vol, seeds, None, step=step, curv_thr=curv_thr,
                    max_steps=max_steps, rng_seed=rng_seed,
                    particles_per_seed=particles_per_seed,
                    recipe="straight tube along x, zero dispersion, F=1, f=1")


# ----------------------------------------------------------------------------- c2

def crossing(nx=64, ny=64, nz=32, lo=24, hi=40, zlo=8, zhi=24, nsamples=50, sigma=0.0,
             f_single=0.7, f_cross=(0.35, 0.35), f_jitter=0.0, nseeds=1000,
             particles_per_seed=5000, step=0.5, max_steps=2000, curv_thr=0.2,
             fib_thr=0.01, gen_seed=12, rng_seed=0x5EED_2012) -> Workload:
    """c2: two bundles crossing at 90 degrees (BASELINE.json configs[1]).

    Bundle A along x (y in [lo,hi), z in [zlo,zhi), all x); bundle B along y
    (x in [lo,hi), z in [zlo,zhi), all y); the 16^3 overlap holds both fibres
    (f = f_cross, fibre 0 = A's direction); elsewhere fibre 1 has f = 0.
    sigma = 0 is the zero-dispersion variant (closed forms, SURVEY C-pin-7); sigma > 0
    the dispersed one.  Seeds: ``nseeds`` distinct mask voxel centres drawn with
    PCG64(gen_seed), sorted in raster order.
    """
    rng = np.random.Generator(np.random.PCG64(gen_seed))
    F, S = 2, nsamples
    dy, f, mask = _empty(nx, ny, nz, S, F)
    A = np.zeros((nz, ny, nx), bool)
    B = np.zeros((nz, ny, nx), bool)
    A[zlo:zhi, lo:hi, :] = True
    B[zlo:zhi, :, lo:hi] = True
    X = A & B
    mask[A | B] = 1
    ex = np.array([1, 0, 0], np.float32)
    ey = np.array([0, 1, 0], np.float32)
    mean0 = np.zeros((nz, ny, nx, 3), np.float32)
    mean0[...] = ex
    mean0[B & ~A] = ey
    mean1 = np.zeros((nz, ny, nx, 3), np.float32)
    mean1[...] = ey
    for s in range(S):
        if sigma > 0:
            dy[0, s] = _disperse(mean0, sigma, rng)
            dy[1, s] = _disperse(mean1, sigma, rng)
        else:
            dy[0, s] = mean0
            dy[1, s] = mean1
        f0 = np.where(X, f_cross[0], np.where(A | B, f_single, 0.0)).astype(np.float32)
        f1 = np.where(X, f_cross[1], 0.0).astype(np.float32)
        if f_jitter > 0:
            f0 = np.where(mask > 0, np.clip(f0 + f_jitter * rng.standard_normal(f0.shape), 0, 1), 0)
            f1 = np.where(X, np.clip(f1 + f_jitter * rng.standard_normal(f1.shape), 0, 1), 0)
        f[0, s] = f0
        f[1, s] = f1
    vol = Volume(nx, ny, nz, S, F, dy, f, mask)
    inside = np.argwhere(mask > 0)[:, ::-1]  # (x, y, z), raster order (x fastest after sort)
    pick = np.sort(rng.choice(inside.shape[0], size=min(nseeds, inside.shape[0]), replace=False))
    order = np.lexsort((inside[pick, 0], inside[pick, 1], inside[pick, 2]))
    seeds = _centres(inside[pick][order])
    return Workload("c2_crossing" + ("_dispersed" if sigma > 0 else ""), vol, seeds, None,
                    step=step, curv_thr=curv_thr, fib_thr=fib_thr, max_steps=max_steps,
                    rng_seed=rng_seed, particles_per_seed=particles_per_seed,
                    recipe=f"90deg crossing, sigma={sigma}, f_jitter={f_jitter}, gen_seed={gen_seed}")


# ----------------------------------------------------------------------------- c3 / c5

def _brain_fields(nx, ny, nz, semi):
    zz, yy, xx = np.meshgrid(np.arange(nz, dtype=np.float32), np.arange(ny, dtype=np.float32),
                             np.arange(nx, dtype=np.float32), indexing="ij")
    cx, cy, cz = (nx - 1) / 2.0, (ny - 1) / 2.0, (nz - 1) / 2.0
    u = (xx - cx) / semi[0]
    v = (yy - cy) / semi[1]
    w = (zz - cz) / semi[2]
    r2 = u * u + v * v + w * w
    # three smooth fibre families: left-right "callosal" arcs in the
    # x-z plane, a superior-inferior "projection" fan from a focus below the brain,
    # an anterior-posterior "association" family along y.
    z0 = cz - 0.9 * semi[2]
    cc = np.stack([-(zz - z0), np.zeros_like(xx), (xx - cx)], -1)
    pr = np.stack([xx - cx, 0.35 * (yy - cy), zz - (cz - 2.2 * semi[2])], -1)
    asn = np.stack([0.12 * np.sin(3.0 * v), np.ones_like(xx), 0.35 * w], -1)
    dirs = [_normalize(cc), _normalize(pr), _normalize(asn)]
    au = np.abs(u)
    wcc = np.exp(-(u / 0.45) ** 2) * (1 / (1 + np.exp(-6 * (w + 0.1)))) + 0.05
    wpr = (1 - np.exp(-(u / 0.30) ** 2)) * np.exp(-((au - 0.30) / 0.30) ** 2) + 0.05
    was = np.exp(-((au - 0.58) / 0.18) ** 2) * np.exp(-(w / 0.55) ** 2) + 0.03
    weights = np.stack([wcc, wpr, was], 0).astype(np.float32)
    s = 0.5 + 0.5 * np.sin(3.1 * u + 1.0) * np.sin(2.7 * v + 2.0) * np.sin(3.3 * w + 0.5)
    sigma = (0.10 + 0.35 * s ** 4).astype(np.float32)
    return r2, dirs, weights, sigma


def whole_brain(nx=128, ny=128, nz=70, nsamples=50, nfibres=2, semi=(58.0, 62.0, 33.0),
                wm_scale=0.8, particles_per_seed=5000, step=0.5, max_steps=2000,
                curv_thr=0.2, fib_thr=0.01, f_total=0.6, cross_ratio=0.62, cross_ratio3=0.40,
                f_jitter=0.03,
                gen_seed=3, rng_seed=0x5EED_2012, seeds: str = "wm") -> Workload:
    """c3 (and c5 with nfibres=3): whole-brain-shaped synthetic volume.

    Brain = ellipsoid with semi-axes ``semi`` (mask); WM = the inner ``wm_scale``
    ellipsoid; WM voxels hold the ``nfibres`` strongest of three smooth families
    (f1 >= f2 >= f3, sum f = f_total, a weaker family is kept only if its weight is
    >= cross_ratio x the strongest), per-sample dispersion sigma(x) in [0.10, 0.45]
    and f jitter 0.03; the GM-like shell holds isotropic samples (uniform on S^2,
    f ~ U(0.05, 0.3)), so the curvature hazard there is ~ curv_thr^F (SURVEY C-pin-9).
    Seeds: every WM voxel centre in raster order (x fastest).
    """
    rng = np.random.Generator(np.random.PCG64(gen_seed))
    F, S = nfibres, nsamples
    r2, dirs, weights, sigma = _brain_fields(nx, ny, nz, semi)
    brain = r2 <= 1.0
    wm = r2 <= wm_scale ** 2
    gm = brain & ~wm
    mask = brain.astype(np.uint8)
    order = np.argsort(-weights, axis=0)  # families by decreasing weight, per voxel
    wsort = np.take_along_axis(weights, order, 0)
    keep = np.zeros_like(wsort, bool)
    keep[0] = True
    for k in range(1, min(F, 3)):
        keep[k] = wsort[k] >= (cross_ratio if k == 1 else cross_ratio3) * wsort[0]
    wk = np.where(keep[:F], wsort[:F], 0.0)
    fmean = (f_total * wk / wk.sum(0, keepdims=True)).astype(np.float32)  # [F][Z][Y][X]
    dmean = np.stack([np.take_along_axis(np.stack(dirs, 0), order[k][None, ..., None].repeat(3, -1), 0)[0]
                      for k in range(F)], 0)  # [F][Z][Y][X][3]
    dy = np.zeros((F, S, nz, ny, nx, 3), np.float32)
    dy[..., 0] = 1.0
    f = np.zeros((F, S, nz, ny, nx), np.float32)
    bidx = np.flatnonzero(brain.ravel())           # only brain voxels get samples
    g_b = gm.ravel()[bidx]
    sig_b = sigma.ravel()[bidx]
    dflat = [dmean[j].reshape(-1, 3)[bidx] for j in range(F)]
    fflat = [fmean[j].ravel()[bidx] for j in range(F)]
    kflat = [keep[j].ravel()[bidx] for j in range(F)]
    ng = int(g_b.sum())
    for s in range(S):
        for j in range(F):
            d = _disperse(dflat[j], sig_b, rng)
            d[g_b] = _normalize(rng.standard_normal((ng, 3), dtype=np.float32))
            dy[j, s].reshape(-1, 3)[bidx] = d
            fj = np.clip(fflat[j] + np.float32(f_jitter) * rng.standard_normal(bidx.size, dtype=np.float32), 0, 1)
            fj = np.where(kflat[j], fj, np.float32(0))
            fj[g_b] = rng.uniform(0.05, 0.3, ng).astype(np.float32)
            f[j, s].reshape(-1)[bidx] = fj
    vol = Volume(nx, ny, nz, S, F, dy, f, mask)
    if seeds == "wm":
        idx = np.argwhere(wm)[:, ::-1]  # argwhere is z-major raster; columns -> (x, y, z)
    else:
        idx = np.argwhere(brain)[:, ::-1]
    name = "c3_whole_brain" if F == 2 and (nx, ny, nz) == (128, 128, 70) else f"brain_{nx}x{ny}x{nz}_F{F}"
    return Workload(name, vol, _centres(idx), None, step=step, curv_thr=curv_thr,
                    fib_thr=fib_thr, max_steps=max_steps, rng_seed=rng_seed,
                    particles_per_seed=particles_per_seed,
                    recipe=f"ellipsoid brain semi={semi}, WM scale {wm_scale}, 3 families, "
                           f"keep ratio {cross_ratio}, gen_seed={gen_seed}")


def wm_seeds(w: Workload, every: int = 1) -> Workload:
    """Every ``every``-th seed of a workload, keeping the global seed ids (for subsets)."""
    ids = w.ids()[::every].copy()
    return w.replace(seeds=w.seeds[::every].copy(), seed_ids=ids)


# ----------------------------------------------------------------------------- pins

def isotropic(n=48, nsamples=4096, nfibres=2, f_value=0.5, nseeds=4, particles_per_seed=5000,
              step=0.5, curv_thr=0.2, max_steps=2000, gen_seed=9, rng_seed=77) -> Workload:
    """All voxels in the mask, samples i.i.d. uniform on S^2, all f > fib_thr (C-pin-9)."""
    rng = np.random.Generator(np.random.PCG64(gen_seed))
    F, S = nfibres, nsamples
    dy = _normalize(rng.standard_normal((F, S, n, n, n, 3), dtype=np.float32))
    f = np.full((F, S, n, n, n), f_value, np.float32)
    mask = np.ones((n, n, n), np.uint8)
    vol = Volume(n, n, n, S, F, dy, f, mask)
    c = n // 2
    seeds = _centres(np.array([[c, c, c]] * nseeds))
    return Workload("isotropic", vol, seeds, None, step=step, curv_thr=curv_thr,
                    max_steps=max_steps, rng_seed=rng_seed, particles_per_seed=particles_per_seed,
                    recipe="isotropic samples")


def bent_tube(c_value: float, nx=32, ny=32, nz=8, x_bend=20, nsamples=8, seed_x=8,
              particles_per_seed=64, curv_thr=0.2, step=0.5, rng_seed=5) -> Workload:
    """C-pin-6: v1 = (1,0,0) for x < x_bend, v2 = (c, s, 0) for x >= x_bend (c = c_value
    as float32, s = sqrt(1-c^2) in float32), mask = whole volume. The fp32 dot of v2 with
    (1,0,0) is exactly c, so the particle ends CURV iff not (c > curv_thr)."""
    F, S = 1, nsamples
    dy, f, mask = _empty(nx, ny, nz, S, F)
    mask[...] = 1
    f[...] = 1.0
    c = np.float32(c_value)
    s = np.float32(math.sqrt(max(0.0, 1.0 - float(c) ** 2)))
    dy[:, :, :, :, x_bend:, :] = np.array([c, s, 0], np.float32)
    vol = Volume(nx, ny, nz, S, F, dy, f, mask)
    seeds = _centres(np.array([[seed_x, ny // 2, nz // 2]]))
    return Workload("bent_tube", vol, seeds, None, step=step, curv_thr=curv_thr,
                    rng_seed=rng_seed, particles_per_seed=particles_per_seed,
                    recipe=f"bent tube c={float(c)!r}")


def fork(after, before=((1.0, 0.0, 0.0), 1.0), nfibres=2, nx=40, ny=40, nz=8, x_bend=20,
         nsamples=4, seed_x=8, particles_per_seed=64, curv_thr=0.2, fib_thr=0.01, step=0.5,
         rng_seed=23) -> Workload:
    """Pins for the fibre choice (R7, R8): for x < x_bend fibre 0 = before[0] with
    f = before[1] (other fibres f = 0); for x >= x_bend the fibres are ``after`` =
    [((vx,vy,vz), f), ...] (float32 values as given).  Mask = whole volume."""
    F, S = nfibres, nsamples
    dy, f, mask = _empty(nx, ny, nz, S, F)
    mask[...] = 1
    dy[0, :, :, :, :x_bend] = np.asarray(before[0], np.float32)
    f[0, :, :, :, :x_bend] = np.float32(before[1])
    for j, (v, fj) in enumerate(after):
        dy[j, :, :, :, x_bend:] = np.asarray(v, np.float32)
        f[j, :, :, :, x_bend:] = np.float32(fj)
    vol = Volume(nx, ny, nz, S, F, dy, f, mask)
    seeds = _centres(np.array([[seed_x, ny // 2, nz // 2]]))
    return Workload("fork", vol, seeds, None, step=step, curv_thr=curv_thr, fib_thr=fib_thr,
                    rng_seed=rng_seed, particles_per_seed=particles_per_seed,
                    recipe=f"fork after x={x_bend}: {after}")


def t_junction(x_j=40, nx=64, ny=64, nz=16, y=(24, 40), width=8, nsamples=16,
               seed_xs=(20, 30), particles_per_seed=200, curv_thr=0.2, step=0.5,
               rng_seed=11) -> Workload:
    """C-pin-7 T-junction: bundle A along x for x < x_j (y in [y0,y1)), then a B-only
    column (fibre (0,1,0), all y) at x in [x_j, x_j+width); F = 2 with f1 = 0 everywhere."""
    F, S = 2, nsamples
    dy, f, mask = _empty(nx, ny, nz, S, F)
    mask[:, y[0]:y[1], :x_j] = 1
    mask[:, :, x_j:x_j + width] = 1
    dy[0] = np.array([1, 0, 0], np.float32)
    dy[0, :, :, :, x_j:x_j + width] = np.array([0, 1, 0], np.float32)
    dy[1] = np.array([0, 0, 1], np.float32)
    f[0] = np.where(mask > 0, 0.7, 0.0)
    vol = Volume(nx, ny, nz, S, F, dy, f, mask)
    seeds = _centres(np.array([[xs, (y[0] + y[1]) // 2, nz // 2] for xs in seed_xs]))
    return Workload("t_junction", vol, seeds, None, step=step, curv_thr=curv_thr,
                    rng_seed=rng_seed, particles_per_seed=particles_per_seed,
                    recipe=f"T junction at x={x_j}")


def vortex(n=48, nz=4, r_in=6.0, r_out=20.0, nsamples=8, sigma=0.0, seed_r=(10, 13, 16), nseeds_per_r=4,
           particles_per_seed=32, max_steps=600, step=0.5, curv_thr=0.2, gen_seed=31, rng_seed=99) -> Workload:
    """Closed loops (NEXT-2 pins, R25): an annulus r_in <= r < r_out around the volume's
    z-axis, F = 1, fibre = the tangent (-dy, dx, 0) / r at the voxel centre (plus a sigma
    dispersion per sample), f = 1, mask = the annulus (all slices).  Streamlines circle the
    axis and come back to voxels they have already entered, so a per-streamline-unique map
    differs from the step map.  Seeds at voxel centres on circles of radius seed_r."""
    rng = np.random.Generator(np.random.PCG64(gen_seed))
    F, S = 1, nsamples
    dy, f, mask = _empty(n, n, nz, S, F)
    zz, yy, xx = np.meshgrid(np.arange(nz), np.arange(n), np.arange(n), indexing="ij")
    cx = cy = n / 2.0
    dxv, dyv = xx + 0.5 - cx, yy + 0.5 - cy
    r = np.sqrt(dxv ** 2 + dyv ** 2)
    mask[(r >= r_in) & (r < r_out)] = 1
    t = np.stack([-dyv, dxv, np.zeros_like(r)], -1) / np.maximum(r, 1e-9)[..., None]
    t = np.broadcast_to(t.astype(np.float32), (F, S, nz, n, n, 3))
    dy[...] = _disperse(t, sigma, rng) if sigma > 0 else t
    f[...] = 1.0
    vol = Volume(n, n, nz, S, F, np.ascontiguousarray(dy), f, mask)
    pts = []
    for rr in seed_r:
        for k in range(nseeds_per_r):
            a = 2 * math.pi * k / nseeds_per_r + 0.3
            pts.append([int(cx + rr * math.cos(a)), int(cy + rr * math.sin(a)), nz // 2])
    seeds = _centres(np.array(pts))
    return Workload("vortex", vol, seeds, None, step=step, curv_thr=curv_thr, max_steps=max_steps,
                    rng_seed=rng_seed, particles_per_seed=particles_per_seed,
                    recipe=f"vortex annulus [{r_in}, {r_out}) sigma {sigma}")


def mirror_x(w: Workload) -> Workload:
    """Mirror a workload in x: voxel (x,y,z) <-> (N-1-x,y,z), v -> (-vx, vy, vz); seeds
    mirrored as x -> N - x (exact for voxel-centre seeds). Same seed ids (C-pin-8)."""
    v = w.volume
    dy = v.dyads[:, :, :, :, ::-1, :].copy()
    dy[..., 0] = -dy[..., 0]
    f = v.f[:, :, :, :, ::-1].copy()
    mask = v.mask[:, :, ::-1].copy()
    seeds = w.seeds.copy()
    seeds[:, 0] = np.float32(v.nx) - seeds[:, 0]
    vol = Volume(v.nx, v.ny, v.nz, v.nsamples, v.nfibres, np.ascontiguousarray(dy),
                 np.ascontiguousarray(f), np.ascontiguousarray(mask))
    return w.replace(name=w.name + "_mirror", volume=vol, seeds=seeds, seed_ids=w.ids())


def to_half(w: Workload) -> Workload:
    """fp16 records (c4): the generator rounds once (numpy RNE), both sides read the halves."""
    v = w.volume
    vol = Volume(v.nx, v.ny, v.nz, v.nsamples, v.nfibres, v.dyads.astype(np.float16),
                 v.f.astype(np.float16), v.mask)
    return w.replace(name=w.name + "_f16", volume=vol)


# ----------------------------------------------------------------------------- paper mode

def paper_dataset(which: int = 1, step: float = 0.1, curv_thr: float = 0.9, gen_seed: int = 21) -> Workload:
    """NEXT-1 workload shaped like the paper's datasets: #1 48x96x96, #2 60x102x102
    (read as 96x96 / 102x102 in-plane, 48 / 60 slices), brain ellipsoid with c3's
    proportions, seeds = every brain voxel ("from each voxel in the brain"),
    50 samples and one streamline per sample volume (P = S = 50, sample_mode 1,
    Alg. 1), MaxStep = sum of the segmentation array = 1888."""
    nx, ny, nz = (96, 96, 48) if which == 1 else (102, 102, 60)
    semi = (0.453 * nx, 0.484 * ny, 0.471 * nz)
    w = whole_brain(nx=nx, ny=ny, nz=nz, semi=semi, nsamples=50, nfibres=2, particles_per_seed=50,
                    step=step, curv_thr=curv_thr, max_steps=1888, gen_seed=gen_seed, seeds="brain")
    return w.replace(name=f"paper_d{which}_step{step}_thr{curv_thr}", sample_mode=1,
                     recipe=w.recipe + f"; paper mode D{which}, step {step}, dot threshold {curv_thr}")


# ----------------------------------------------------------------------------- NEXT-4 DWI

@dataclasses.dataclass
class DwiWorkload:
    """Synthetic diffusion-weighted data for the MCMC sampler (NEXT-4, Fig. 1: a 4-D
    volume of n measurements, b-values and gradient directions) plus the sampler settings."""
    name: str
    nx: int
    ny: int
    nz: int
    dwi: np.ndarray       # [n][Z][Y][X] float32
    bvals: np.ndarray     # [n] float32 (ms/um^2: b = 1 is 1000 s/mm^2)
    bvecs: np.ndarray     # [n][3] float32 unit vectors
    mask: np.ndarray      # [Z][Y][X] uint8: voxels to sample ("valid (white matter)")
    truth: Optional[np.ndarray] = None  # [NP][Z][Y][X] float64 generating parameters
    nfibres: int = 2      # N = 2
    burnin: int = 500     # NumBurnIn
    nsamples: int = 50
    interval: int = 2     # L
    adapt_every: int = 50  # K (Fig. 2; reading M8)
    rng_seed: int = 0x4D434D43_2012
    recipe: str = ""

    @property
    def nmeas(self) -> int:
        return int(self.bvals.size)

    @property
    def nvoxels(self) -> int:
        return int((self.mask != 0).sum())

    @property
    def nparams(self) -> int:
        return 3 + 3 * self.nfibres

    @property
    def loops(self) -> int:
        return self.burnin + self.nsamples * self.interval

    def replace(self, **kw) -> "DwiWorkload":
        return dataclasses.replace(self, **kw)


def gradient_scheme(ndirs: int = 60, nb0: int = 4, b: float = 1.0):
    """nb0 b = 0 measurements followed by ndirs directions on the upper hemisphere
    (Fibonacci lattice), all at b.  Returns (bvals [n] float32, bvecs [n][3] float32)."""
    k = np.arange(ndirs, dtype=np.float64) + 0.5
    z = 1.0 - k / ndirs                       # (0, 1]: upper hemisphere
    phi = k * math.pi * (3.0 - math.sqrt(5.0))
    rr = np.sqrt(1.0 - z * z)
    dirs = np.stack([rr * np.cos(phi), rr * np.sin(phi), z], 1)
    bvecs = np.concatenate([np.tile([[1.0, 0.0, 0.0]], (nb0, 1)), dirs], 0).astype(np.float32)
    bvals = np.concatenate([np.zeros(nb0), np.full(ndirs, b)]).astype(np.float32)
    return bvals, bvecs


def _forward(S0, d, f, v, bvals, bvecs):
    """Synthetic scanner: the multiple partial volume model of Eq. 1, numpy
    float64 over voxels.  S0, d: [m]; f: [N][m]; v: [N][m][3]; returns [n][m]."""
    b = bvals.astype(np.float64)[:, None]
    r = bvecs.astype(np.float64)
    att = (1.0 - f.sum(0))[None, :] * np.exp(-b * d[None, :])
    for j in range(f.shape[0]):
        dot = r @ v[j].T                      # [n][m]
        att = att + f[j][None, :] * np.exp(-b * d[None, :] * dot * dot)
    return S0[None, :] * att


def dwi_brain(nx=102, ny=102, nz=60, nfibres=2, scale=1.0803, snr=25.0, ndirs=60, nb0=4, b=1.0,
              gen_seed=41, **kw) -> DwiWorkload:
    """NEXT-4 workload: brain-shaped DWI (the c3 fibre families, ``_brain_fields``).  Mask
    = an ellipsoid of semi-axes scale x half the box (clipped to the box), sized so the
    valid-voxel count matches Table III: 102x102x60 -> ~402k (dataset 2),
    96x96x48 -> ~205k (dataset 1).  Ground truth per voxel: the N strongest families with
    f_total 0.6 (as c3), S0 = 1000 (1 + 0.05 g), d = 1.0 (1 + 0.1 g) um^2/ms; Gaussian noise
    sigma = S0 / snr.  Gradient scheme: ``gradient_scheme(ndirs, nb0, b)``."""
    rng = np.random.Generator(np.random.PCG64(gen_seed))
    semi = (scale * nx / 2.0, scale * ny / 2.0, scale * nz / 2.0)
    r2, dirs, weights, _ = _brain_fields(nx, ny, nz, semi)
    mask = (r2 <= 1.0).astype(np.uint8)
    V = nx * ny * nz
    idx = np.flatnonzero(mask.ravel())
    m = idx.size
    N = nfibres
    order = np.argsort(-weights, axis=0).reshape(3, -1)[:, idx]
    wsort = np.take_along_axis(weights.reshape(3, -1)[:, idx], order, 0)
    keep = np.zeros_like(wsort, bool)
    keep[0] = True
    for k in range(1, min(N, 3)):
        keep[k] = wsort[k] >= (0.62 if k == 1 else 0.40) * wsort[0]
    wk = np.where(keep[:N], wsort[:N], 0.0)
    f = 0.6 * wk / wk.sum(0, keepdims=True)
    fam = np.stack([dd.reshape(-1, 3)[idx] for dd in dirs], 0).astype(np.float64)   # [3][m][3]
    v = np.stack([np.take_along_axis(fam, order[k][None, :, None].repeat(3, -1), 0)[0] for k in range(N)], 0)
    S0 = 1000.0 * (1.0 + 0.05 * rng.standard_normal(m))
    d = 1.0 * (1.0 + 0.1 * rng.standard_normal(m))
    bvals, bvecs = gradient_scheme(ndirs, nb0, b)
    mu = _forward(S0, d, f, v, bvals, bvecs)
    y = mu + (S0 / snr)[None, :] * rng.standard_normal(mu.shape)
    dwi = np.zeros((bvals.size, V), np.float32)
    dwi[:, idx] = y.astype(np.float32)
    NP = 3 + 3 * N
    truth = np.zeros((NP, V), np.float64)
    truth[0, idx] = S0
    truth[1, idx] = d
    truth[2, idx] = S0 / snr
    for j in range(N):
        vj = v[j] * np.where(v[j][:, 2:3] < 0, -1.0, 1.0)      # theta in [0, pi/2]
        truth[3 + 3 * j, idx] = f[j]
        truth[4 + 3 * j, idx] = np.arccos(np.clip(vj[:, 2], -1, 1))
        truth[5 + 3 * j, idx] = np.arctan2(vj[:, 1], vj[:, 0])
    return DwiWorkload(f"dwi_brain_{nx}x{ny}x{nz}_N{N}", nx, ny, nz,
                       np.ascontiguousarray(dwi.reshape(bvals.size, nz, ny, nx)), bvals, bvecs,
                       np.ascontiguousarray(mask), truth.reshape(NP, nz, ny, nx), nfibres=N,
                       recipe=f"brain ellipsoid scale {scale}, {m} voxels, SNR {snr}, "
                              f"{nb0} b0 + {ndirs} dirs at b={b}, gen_seed={gen_seed}", **kw)


def dwi_uniform(nvox=64, S0=1000.0, d=1.0, f=(0.4, 0.2), v=((1.0, 0.0, 0.0), (0.0, 1.0, 0.0)),
                snr=25.0, ndirs=60, nb0=4, b=1.0, gen_seed=5, nx=None, **kw) -> DwiWorkload:
    """nvox voxels (a 1-row volume, all in the mask) with the same generating parameters and
    independent noise: the pins' workload (posterior statistics across voxels)."""
    rng = np.random.Generator(np.random.PCG64(gen_seed))
    N = len(f)
    bvals, bvecs = gradient_scheme(ndirs, nb0, b)
    vv = np.array([np.asarray(x, np.float64) / np.linalg.norm(x) for x in v])[:, None, :].repeat(nvox, 1)
    S0a = np.full(nvox, float(S0))
    da = np.full(nvox, float(d))
    fa = np.array([np.full(nvox, float(x)) for x in f])
    mu = _forward(S0a, da, fa, vv, bvals, bvecs)
    y = mu + (S0 / snr) * rng.standard_normal(mu.shape) if snr else mu
    nx = nvox if nx is None else nx
    NP = 3 + 3 * N
    truth = np.zeros((NP, nvox))
    truth[0] = S0
    truth[1] = d
    truth[2] = S0 / snr if snr else 0.0
    for j in range(N):
        truth[3 + 3 * j] = f[j]
        truth[4 + 3 * j] = math.acos(max(-1.0, min(1.0, vv[j, 0, 2])))
        truth[5 + 3 * j] = math.atan2(vv[j, 0, 1], vv[j, 0, 0])
    return DwiWorkload(f"dwi_uniform_{nvox}", nx, 1, 1,
                       np.ascontiguousarray(y.astype(np.float32).reshape(bvals.size, 1, 1, nx)), bvals, bvecs,
                       np.ones((1, 1, nx), np.uint8), truth.reshape(NP, 1, 1, nx), nfibres=N,
                       recipe=f"uniform voxels S0={S0} d={d} f={f} snr={snr}", **kw)


MCMC_CONFIGS = {
    # Table III shapes: valid-voxel counts ~205k / ~402k
    "m1": lambda: dwi_brain(96, 96, 48, scale=0.96, gen_seed=43),
    "m2": lambda: dwi_brain(102, 102, 60, scale=1.0803, gen_seed=41),
    "m_small": lambda: dwi_brain(24, 24, 16, scale=1.0, gen_seed=47, burnin=100, nsamples=10),
    # profiling subset of m2 (every 8th valid voxel): same per-voxel work, 1/8 of the voxels
    "m2_prof": lambda: mcmc_subset(dwi_brain(102, 102, 60, scale=1.0803, gen_seed=41), 8),
}


def mcmc_subset(d: DwiWorkload, every: int) -> DwiWorkload:
    """Every ``every``-th valid voxel of a DWI workload (profiling / CPU samples)."""
    m = d.mask.ravel().copy()
    idx = np.flatnonzero(m)
    m[:] = 0
    m[idx[::every]] = 1
    return d.replace(mask=m.reshape(d.mask.shape), name=d.name + f"_every{every}")


def mcmc_config(name: str) -> DwiWorkload:
    return MCMC_CONFIGS[name]()


# ----------------------------------------------------------------------------- configs

CONFIGS = {
    # BASELINE.json configs[i] -> generator call (full size)
    "c1": lambda: tube(),
    "c2": lambda: crossing(),
    "c2_dispersed": lambda: crossing(sigma=0.15, f_jitter=0.03),
    "c3": lambda: whole_brain(),
    "c4": lambda: to_half(whole_brain()),
    "c5": lambda: to_half(whole_brain(nx=145, ny=174, nz=145, nfibres=3,
                                      semi=(66.0, 82.0, 66.0), particles_per_seed=10000)),
    # NEXT-1: the paper's own mode on dataset-shaped phantoms (Table II parameters)
    "d1": lambda: paper_dataset(1, 0.1, 0.9),
    "d1_s02": lambda: paper_dataset(1, 0.2, 0.8),
    "d1_s03": lambda: paper_dataset(1, 0.3, 0.85),
    "d2": lambda: paper_dataset(2, 0.1, 0.9),
    "d2_s02": lambda: paper_dataset(2, 0.2, 0.85),
    "d2_s03": lambda: paper_dataset(2, 0.3, 0.8),
}


def config(name: str) -> Workload:
    w = CONFIGS[name]()
    w.volume.check()
    return w
