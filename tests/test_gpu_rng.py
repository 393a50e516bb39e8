"""Device side of the frozen RNG contract (``-m gpu``): the tracking kernel's own Philox and
sample-index functions (pt_rng_draws, the same device code the stepping kernel inlines)
reproduce tests/golden/rng_draws.txt -- written from the oracle alone -- and agree with the
CUDA library's curand_Philox4x32_10 on every block (SURVEY C-pin-1)."""
from __future__ import annotations

import numpy as np
import pytest

from tests.test_rng_contract import KEY, rows

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tracker():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_ipps_xuzwrwxgxy12_b200 as pt
    pt.build()
    t = pt.Tracker(0)
    yield t
    t.close()


def test_device_rng_reproduces_golden(tracker):
    r = np.array(rows(), dtype=object)
    pid = np.array([int(x) for x in r[:, 0]], np.uint64)
    stream = r[:, 1].astype(np.uint32)
    block = r[:, 3].astype(np.uint32)
    expect_w = r[:, 5:9].astype(np.uint64).astype(np.uint32)
    for S in sorted({int(x) for x in r[:, 9]}):
        sel = r[:, 9].astype(int) == S
        words, samples, mism = tracker.rng_draws(pid[sel], block[sel], stream[sel], KEY, S)
        assert mism == 0
        assert np.array_equal(words, expect_w[sel])
        word = r[sel, 4].astype(int)
        s = r[sel, 10].astype(int)
        k = word >= 0
        got = samples[np.arange(sel.sum())[k], word[k]].astype(int)
        assert np.array_equal(got, s[k])


def test_device_rng_matches_curand_at_scale(tracker):
    rng = np.random.default_rng(7)
    n = 1 << 20
    pid = rng.integers(0, 2**63, n, dtype=np.int64).astype(np.uint64) * np.uint64(2) + rng.integers(0, 2, n).astype(np.uint64)
    block = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
    stream = rng.integers(0, 4, n).astype(np.uint32)
    words, samples, mism = tracker.rng_draws(pid, block, stream, 0xDEADBEEFCAFEF00D, 50)
    assert mism == 0
    assert np.array_equal(samples, ((words[:, :3].astype(np.uint64) * np.uint64(50)) >> np.uint64(32)).astype(np.uint32))
