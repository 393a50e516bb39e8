"""The oracle under AddressSanitizer + UndefinedBehaviorSanitizer (SURVEY §5 sanitizers):
an ASan/UBSan build of oracle.c + oracle_mcmc.c runs every code path the tests use -- the
base contract, paths, connectivity, the unique map, the NEXT-3 variants, paper mode, edge
seeds, fp16 records, and the MCMC sampler -- in a child Python with libasan preloaded.
Any out-of-bounds access, use-after-free, leak-free misuse or UB (signed overflow, bad
shift, misaligned load) aborts the child.  CPU only."""
from __future__ import annotations

import os
import subprocess
import sys

import pytest

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import numpy as np
import oracle, phantom
w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=12, particles_per_seed=12, nsamples=8)
edge = np.array([[-5.0, 3.0, 3.0], [0.5, 0.5, 0.5], [70.0, 1.0, 1.0], [np.nan, 1, 1]], np.float32)
w = w.replace(seeds=np.concatenate([w.seeds, edge]))
lab = (np.arange(w.volume.mask.size).reshape(w.volume.mask.shape) % 7).astype(np.uint8)
for kw in ({}, {"bidir": 1}, {"interp": 1, "init_fibre": 2}, {"bidir": 1, "interp": 1, "init_fibre": 1},
           {"sample_mode": 1}, {"max_steps": 1}):
    ww = w.replace(**kw)
    oracle.track(ww, path_stride=17, labels=lab, ntargets=6, want_unique=True)
    oracle.track(phantom.to_half(ww), want_unique=True, threads=2)
b = phantom.whole_brain(nx=16, ny=14, nz=10, semi=(7.0, 6.0, 4.0), nsamples=6, nfibres=3, particles_per_seed=5,
                        seeds="brain")
oracle.track(phantom.wm_seeds(b, every=5), path_stride=9, want_unique=True)
d = phantom.dwi_uniform(nvox=6, burnin=10, nsamples=3, interval=2, adapt_every=5)
oracle.mcmc(d)
print("SANITIZED-OK")
'''


def test_oracle_asan_ubsan(tmp_path):
    asan = subprocess.run(["gcc", "-print-file-name=libasan.so"], capture_output=True, text=True).stdout.strip()
    if not os.path.isabs(asan) or not os.path.exists(asan):
        pytest.skip("libasan not available")
    lib = oracle.build(out=str(tmp_path / "liboracle_san.so"), sanitize=True, force=True)
    env = dict(os.environ, LD_PRELOAD=asan, ORACLE_LIB=lib, PYTHONPATH=ROOT,
               ASAN_OPTIONS="detect_leaks=0:abort_on_error=1", UBSAN_OPTIONS="print_stacktrace=1")
    out = subprocess.run([sys.executable, "-c", CHILD], capture_output=True, text=True, timeout=900, cwd=ROOT,
                         env=env)
    assert out.returncode == 0, out.stderr[-4000:]
    assert "SANITIZED-OK" in out.stdout
    assert "runtime error" not in out.stderr and "AddressSanitizer" not in out.stderr
