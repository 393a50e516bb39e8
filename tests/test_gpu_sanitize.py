"""compute-sanitizer on the tracking kernels (SURVEY §5 sanitizers; ``-m gpu``).

memcheck (out-of-bounds / misaligned device accesses, leaks of device allocations),
racecheck (shared-memory hazards: the CTA claim / ticket word and the per-warp sub-chunk
slots of pt_claim.cuh) and synccheck (barrier misuse) over small configs through every
kernel: the persistent round kernel with and without outputs, the variant and unique-map
instantiations, the no-refill and segmented ablations, targets, paths, MCMC.  The child
uses the C ABI with host numpy buffers only (no torch), so the sanitizer sees our kernels
and the CUDA runtime, nothing else."""
from __future__ import annotations

import os
import re
import shutil
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu

CHILD = r'''
import ctypes, numpy as np
import paper_conf_ipps_xuzwrwxgxy12_b200 as pt, phantom
ctx = pt.pt_create(0)
def load(w):
    v = w.volume
    pt.pt_load_samples(ctx, v.nx, v.ny, v.nz, v.nsamples, v.nfibres, pt.PT_F16 if v.is_half else pt.PT_F32,
                       v.dyads.ctypes.data, v.f.ctypes.data, v.mask.ctypes.data)
def track(w, flags, stride=0):
    prm = pt.pt_params(w.step, w.curv_thr, w.fib_thr, w.max_steps, w.rng_seed, w.particles_per_seed, flags, stride)
    m = np.zeros(w.volume.mask.shape, np.uint32)
    ids = w.ids()
    pt.pt_track(ctx, w.seeds.ctypes.data, ids.ctypes.data, w.nseeds, prm, m.ctypes.data)
    n = w.nparticles * (2 if flags & pt.PT_BIDIR else 1)
    if flags & (pt.PT_REC_LEN | pt.PT_REC_REASON | pt.PT_REC_END | pt.PT_REC_PATHS):
        q = pt.pt_paths()
        q.capacity = n
        a = np.zeros(n, np.uint16); b = np.zeros(n, np.uint8); e = np.zeros((n, 3), np.float32)
        p = np.zeros((n, max(stride, 1), 3), np.float32)
        q.nsteps = a.ctypes.data if flags & pt.PT_REC_LEN else None
        q.reason = b.ctypes.data if flags & pt.PT_REC_REASON else None
        q.end_xyz = e.ctypes.data if flags & pt.PT_REC_END else None
        q.paths = p.ctypes.data if flags & pt.PT_REC_PATHS else None
        pt.pt_get_paths(ctx, q)
    pt.pt_get_stats(ctx)
    return m
REC = pt.PT_REC_LEN | pt.PT_REC_REASON | pt.PT_REC_END
w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=24, particles_per_seed=40, nsamples=8)
w = w.replace(seeds=np.concatenate([w.seeds, np.array([[-5, 3, 3], [0.5, 0.5, 0.5]], np.float32)]))
for ww in (w, phantom.to_half(w)):
    load(ww)
    for fl in (0, REC, REC | pt.PT_REC_PATHS, REC | pt.PT_KERNEL_SIMPLE, REC | pt.PT_KERNEL_SEGMENTED,
               REC | pt.PT_KERNEL_VARIANT, REC | pt.PT_BIDIR | pt.PT_INTERP | pt.PT_INIT_FWEIGHT,
               pt.PT_BIDIR | pt.PT_INIT_RANDOM, pt.PT_MAP_UNIQUE, REC | pt.PT_MAP_UNIQUE | pt.PT_BIDIR | pt.PT_INTERP):
        track(ww, fl, 33 if fl & pt.PT_REC_PATHS else 0)
lab = (np.arange(w.volume.mask.size).reshape(w.volume.mask.shape) % 5).astype(np.uint8)
load(w)
pt.pt_load_targets(ctx, lab.ctypes.data, 4)
track(w, REC | pt.PT_REC_CONN)
track(w.replace(particles_per_seed=1, max_steps=3), REC | pt.PT_REC_CONN | pt.PT_BIDIR)
b = phantom.whole_brain(nx=24, ny=20, nz=14, semi=(10.0, 8.0, 5.0), nsamples=6, nfibres=3, particles_per_seed=64)
b = phantom.wm_seeds(b, every=max(1, b.nseeds // 60))
load(b)
track(b, 0)
track(b, REC | pt.PT_MAP_UNIQUE)
d = phantom.dwi_uniform(nvox=8, burnin=10, nsamples=2, interval=2, adapt_every=5)
sh = pt.pt_dwi_shape(d.nx, d.ny, d.nz, d.bvals.size)
mp = pt.pt_mcmc_params(d.nfibres, d.burnin, d.nsamples, d.interval, d.adapt_every, d.rng_seed, 0)
out = np.zeros((d.nparams, d.nsamples, d.nz, d.ny, d.nx), np.float64)
pt.pt_mcmc(ctx, sh, d.dwi.ctypes.data, d.bvals.ctypes.data, d.bvecs.ctypes.data, d.mask.ctypes.data, mp, None,
           out.ctypes.data, None)
pt.pt_get_mcmc_stats(ctx)
pt.pt_destroy(ctx)
print("SANITIZED-OK")
'''


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    cs = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    if not os.path.exists(cs):
        pytest.skip("compute-sanitizer not found")
    import paper_conf_ipps_xuzwrwxgxy12_b200 as pt
    pt.build()
    extra = ["--leak-check", "full"] if tool == "memcheck" else []
    cmd = [cs, "--tool", tool, "--error-exitcode", "99", *extra, sys.executable, "-c", CHILD]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=1500, cwd=ROOT,
                         env=dict(os.environ, PYTHONPATH=ROOT))
    tail = (out.stdout + out.stderr)[-4000:]
    if "closed on this pool" in tail:  # the pool's wrapper refuses: test_gpu_bounds.py stands in
        pytest.skip("compute-sanitizer is not run on this GPU pool (see tests/test_gpu_bounds.py)")
    assert out.returncode == 0, tail
    assert "SANITIZED-OK" in out.stdout
    text = out.stdout + out.stderr
    assert re.search(r"(ERROR SUMMARY: 0 errors|RACECHECK SUMMARY: 0 hazards)", text), tail
