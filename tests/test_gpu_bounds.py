"""Bounds-checked build of libpt.so (SURVEY §5 sanitizers; ``-m gpu``).

compute-sanitizer is not available on the GPU pool this repo is measured on (its wrapper
refuses to run, see tests/test_gpu_sanitize.py), so memory safety of the kernels is
checked by a build of our own: ``-DPT_CHECK_BOUNDS=1`` compiles a check of every record
gather, map / hash-set / mask / label RED or load, per-particle output and path write,
seed / order / id read of the tracking kernels (persistent round kernel with and without
outputs, variant and unique-map instantiations, the no-refill and segmented ablations)
and of the MCMC kernel against the size of its buffer; a violation sets a device flag
and pt_get_stats / pt_get_mcmc_stats fail with PT_ERR_CUDA.  The workload is the one the
sanitizer test ran (every kernel and mode, fp32 and fp16 records, edge seeds outside the
volume, targets, F = 3 bricks with ragged edges, MCMC).  A negative control
(PT_CHECK_BOUNDS_SHRINK: the buffers are declared half their size) proves the checks fire."""
from __future__ import annotations

import os
import subprocess
import sys

import pytest

from tests.test_gpu_sanitize import CHILD

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bounds_lib(tmp_path_factory):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    lib = str(tmp_path_factory.mktemp("bounds") / "libpt_bounds.so")
    env = dict(os.environ, PT_LIB=lib, PT_NVCC_EXTRA="-DPT_CHECK_BOUNDS=1", PYTHONPATH=ROOT)
    subprocess.run([sys.executable, "-c", "from paper_conf_ipps_xuzwrwxgxy12_b200 import _build; _build.build(force=True)"],
                   check=True, cwd=ROOT, env=env, timeout=1200)
    assert os.path.exists(lib)
    return lib


def _run(lib, **extra):
    env = dict(os.environ, PT_LIB=lib, PYTHONPATH=ROOT, **extra)
    return subprocess.run([sys.executable, "-c", CHILD], capture_output=True, text=True, timeout=1200, cwd=ROOT, env=env)


def test_bounds_checked_build_is_clean(bounds_lib):
    out = _run(bounds_lib)
    assert out.returncode == 0, (out.stdout + out.stderr)[-4000:]
    assert "SANITIZED-OK" in out.stdout


def test_bounds_check_fires_on_shrunk_buffers(bounds_lib):
    out = _run(bounds_lib, PT_CHECK_BOUNDS_SHRINK="1")
    assert out.returncode != 0
    assert "bounds check (PT_CHECK_BOUNDS build)" in out.stderr + out.stdout
