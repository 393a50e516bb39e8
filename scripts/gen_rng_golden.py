"""Write tests/golden/rng_draws.txt: the frozen tracking-RNG contract (R16) as a
table of draws, computed by the ORACLE only (oracle.philox / oracle.sample_index).

Each row: pid stream n block word w0 w1 w2 w3 S s sign
  block = n // 3 and word = n % 3 for the sample index of step n (streams 0 and 1, R16/R22);
  s = floor(w[word] * S / 2^32); sign = top bit of w3 (meaningful for block 0 of stream 0,
  the first step's sign, R6).  Streams 2 and 3 rows use block = n (R23/R24), word = -1.
Run: python scripts/gen_rng_golden.py  (re-running must reproduce the committed file)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402

KEY = 0x5EED_2012  # phantom.Workload.rng_seed default
rng = np.random.Generator(np.random.PCG64(16))
pids = [0, 1, 2, 4999, 5000, 2**32 - 1, 2**32, 2**32 + 1, 2**33 + 12345, 2**63 + 7, 2**64 - 1]
pids += [int(x) for x in rng.integers(0, 2**63, 25, dtype=np.int64)]
ns = [0, 1, 2, 3, 4, 5, 6, 7, 11, 12, 1887, 1999, 65534]
S_list = [50, 1, 7, 4096]
rows = []
for i, pid in enumerate(pids):
    for stream in (0, 1, 2, 3):
        for n in (ns if stream < 2 else [0, 1, 5, 1999]):
            if (i + n + stream) % 3 == 2 and n not in (0, 1):
                continue  # thin the table: ~200 rows in total
            S = S_list[(i + n) % len(S_list)]
            if stream < 2:
                block, word = n // 3, n % 3
            else:
                block, word = n, -1
            w = oracle.philox([block, pid & 0xFFFFFFFF, pid >> 32, stream], [KEY & 0xFFFFFFFF, KEY >> 32])
            s = oracle.sample_index(int(w[word]), S) if word >= 0 else -1
            rows.append((pid, stream, n, block, word, *[int(x) for x in w], S, s, int(w[3]) >> 31))
out = os.path.join(ROOT, "tests", "golden", "rng_draws.txt")
with open(out, "w") as fh:
    fh.write("# Frozen tracking-RNG contract (DESIGN.md R16), written by scripts/gen_rng_golden.py from\n")
    fh.write(f"# oracle/ only.  key = 0x{KEY:x}; counter = {{block, lo32(pid), hi32(pid), stream}}.\n")
    fh.write("# pid stream n block word w0 w1 w2 w3 S s sign\n")
    for r in rows:
        fh.write(" ".join(str(x) for x in r) + "\n")
print(out, len(rows))
