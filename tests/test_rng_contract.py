"""The frozen tracking-RNG contract (R16; the paper has no tracking RNG -- its
combined Tausworthe generator, draws the MCMC proposals -- so the layout is a free
convention, fixed once and for all by tests/golden/rng_draws.txt).  CPU only.

The golden table was written by scripts/gen_rng_golden.py from oracle/ alone.  Here it is
checked against (a) the oracle as it stands (any later edit of the oracle's RNG use fails),
(b) the independent pure-Python Philox of tests/bruteforce.py, (c) the integer mappings
written out (s = floor(w S / 2^32), sign = top bit), and (d) the Random123 KAT (in
test_oracle_pins.py).  The GPU side is checked against the same table in test_gpu_rng.py."""
from __future__ import annotations

import os

import pytest

import oracle
from tests import bruteforce

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "rng_draws.txt")
KEY = 0x5EED_2012


def rows():
    out = []
    for line in open(GOLDEN):
        if line.startswith("#") or not line.strip():
            continue
        out.append([int(x) for x in line.split()])
    return out


def test_golden_table_shape():
    r = rows()
    assert len(r) >= 200
    streams = {x[1] for x in r}
    assert streams == {0, 1, 2, 3}
    # edge pids (32-bit carry, 2^64 - 1) and edge steps are present
    pids = {x[0] for x in r}
    assert {0, 2**32 - 1, 2**32, 2**64 - 1} <= pids
    assert {0, 1, 2, 3, 65534} <= {x[2] for x in r if x[1] == 0}


def test_oracle_reproduces_golden():
    key = [KEY & 0xFFFFFFFF, KEY >> 32]
    for pid, stream, n, block, word, w0, w1, w2, w3, S, s, sign in rows():
        w = oracle.philox([block, pid & 0xFFFFFFFF, pid >> 32, stream], key)
        assert [int(v) for v in w] == [w0, w1, w2, w3], (pid, stream, n)
        if word >= 0:
            assert oracle.sample_index([w0, w1, w2][word], S) == s


def test_counter_layout_and_mappings():
    """(c): the contract written out in Python integers, and (b) a third Philox."""
    key = (KEY & 0xFFFFFFFF, KEY >> 32)
    for pid, stream, n, block, word, w0, w1, w2, w3, S, s, sign in rows():
        if stream < 2:
            assert block == n // 3 and word == n % 3
            assert s == ([w0, w1, w2][word] * S) >> 32 and 0 <= s < S
        else:
            assert block == n and word == -1
        assert sign == w3 >> 31
        assert list(bruteforce.philox4x32_10([block, pid & 0xFFFFFFFF, pid >> 32, stream], key)) == [w0, w1, w2, w3]


@pytest.mark.parametrize("seed", [1, 2])
def test_golden_regenerates_identically(seed, tmp_path):
    """The committed table is exactly what the generator script writes."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    before = open(GOLDEN).read()
    subprocess.check_call([sys.executable, os.path.join(root, "scripts", "gen_rng_golden.py")],
                          stdout=subprocess.DEVNULL)
    assert open(GOLDEN).read() == before
