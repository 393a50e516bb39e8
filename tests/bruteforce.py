"""Third, independent tracker (SURVEY C-pin-11): numpy float32 scalars, Python-int Philox.

Used only to pin the oracle on tiny inputs: per-step positions must be bit-identical.
It shares nothing with ``oracle/`` (different language, own Philox, own fp16 decode via
numpy's float16 -> float32 cast, own lookup) and nothing with the CUDA path.  numpy
float32 scalar arithmetic is single-rounded binary32 (NEP 50) and never fused.
"""
from __future__ import annotations

import numpy as np

_M = 0xFFFFFFFF


def philox4x32_10(ctr, key):
    c = [int(x) & _M for x in ctr]
    k0, k1 = int(key[0]) & _M, int(key[1]) & _M
    for r in range(10):
        if r:
            k0 = (k0 + 0x9E3779B9) & _M
            k1 = (k1 + 0xBB67AE85) & _M
        p0 = 0xD2511F53 * c[0]
        p1 = 0xCD9E8D57 * c[2]
        c = [((p1 >> 32) ^ c[1] ^ k0) & _M, p1 & _M, ((p0 >> 32) ^ c[3] ^ k1) & _M, p0 & _M]
    return c


def _axis(q: np.float32, n: int) -> int:
    c = n // 2
    if not abs(float(q)) < 1e9:
        return -1
    return c + int(np.trunc(q)) - (1 if np.signbit(q) else 0)


def track(w, seed_index: int, j: int, max_points: int = 10**9):
    """Track one particle; returns (nsteps, reason, positions float32 [n+1][3])."""
    v = w.volume
    dy = v.dyads.astype(np.float32)
    fr = v.f.astype(np.float32)
    F, S = v.nfibres, v.nsamples
    N = (v.nx, v.ny, v.nz)
    c = [np.float32(n // 2) for n in N]
    sid = int(w.ids()[seed_index])
    P = int(w.particles_per_seed)
    pid = sid * P + j
    key = (w.rng_seed & _M, w.rng_seed >> 32)
    h = np.float32(w.step)
    thr = np.float32(w.curv_thr)
    fthr = np.float32(w.fib_thr)

    def lookup(q):
        ix, iy, iz = (_axis(q[a], N[a]) for a in range(3))
        if not (0 <= ix < N[0] and 0 <= iy < N[1] and 0 <= iz < N[2]):
            return None
        if v.mask[iz, iy, ix] == 0:
            return None
        return (iz, iy, ix)

    q = [np.float32(w.seeds[seed_index][a]) - c[a] for a in range(3)]
    pos = [[q[a] + c[a] for a in range(3)]]
    vox = lookup(q)
    if vox is None:
        return 0, 0, np.array(pos, np.float32)
    n = 0
    p = None
    while True:
        if n == w.max_steps:
            return n, 2, np.array(pos, np.float32)
        wd = philox4x32_10([n // 3, pid & _M, pid >> 32, 0], key)
        s = (j % S) if getattr(w, "sample_mode", 0) == 1 else (wd[n % 3] * S) >> 32
        vv = [[dy[jj, s, vox[0], vox[1], vox[2], a] for a in range(3)] for jj in range(F)]
        ff = [fr[jj, s, vox[0], vox[1], vox[2]] for jj in range(F)]
        if n == 0:
            js = 0
            sg = np.float32(-1.0) if (wd[3] >> 31) else np.float32(1.0)
        else:
            dots = [(vv[jj][0] * p[0] + vv[jj][1] * p[1]) + vv[jj][2] * p[2] for jj in range(F)]
            js = None
            for jj in range(F):
                if ff[jj] > fthr and (js is None or abs(dots[jj]) > abs(dots[js])):
                    js = jj
            if js is None:
                js = 0
            if not (abs(dots[js]) > thr):
                return n, 1, np.array(pos, np.float32)
            sg = np.float32(1.0) if dots[js] > np.float32(0) else np.float32(-1.0)
        d = [sg * vv[js][a] for a in range(3)]
        qn = [q[a] + h * d[a] for a in range(3)]
        vn = lookup(qn)
        if vn is None:
            return n, 0, np.array(pos, np.float32)
        q, p, vox = qn, d, vn
        n += 1
        if len(pos) < max_points:
            pos.append([q[a] + c[a] for a in range(3)])
