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


def _interp_voxel(q, wi, N, mask):
    """R23 restated: per axis the upper of the two voxels whose centres bracket q is taken
    with probability = its linear weight; None if outside the volume or the mask."""
    idx = []
    for a in range(3):
        t = np.float32(q[a]) - np.float32(0.5)
        m = np.floor(t)
        fr = t - m
        r = np.float32(wi[a] >> 8) * np.float32(2.0 ** -24)
        k = N[a] // 2 + int(m) + (1 if r < fr else 0)
        if not 0 <= k < N[a]:
            return None
        idx.append(k)
    if mask[idx[2], idx[1], idx[0]] == 0:
        return None
    return (idx[2], idx[1], idx[0])


def _first_fibre(mode, ff, fthr, word):
    """R24 restated: eligible = f > fib_thr; 0 first, 1 uniform, 2 f-weighted."""
    el = [jj for jj in range(len(ff)) if ff[jj] > fthr]
    if mode == 0 or not el:
        return 0
    if mode == 1:
        return el[(word * len(el)) >> 32]
    tot = np.float32(0)
    for jj in el:
        tot = tot + ff[jj]
    r = (np.float32(word >> 8) * np.float32(2.0 ** -24)) * tot
    cum = np.float32(0)
    for jj in el:
        cum = cum + ff[jj]
        if r < cum:
            return jj
    return el[-1]


def track(w, seed_index: int, j: int, max_points: int = 10**9):
    """Track one particle (half 0); returns (nsteps, reason, positions float32 [n+1][3])."""
    n, why, pos, _, _ = _half(w, seed_index, j, 0, None, max_points)
    return n, why, pos


def streamline_voxels(w, seed_index: int, j: int) -> set:
    """The set of voxels (z, y, x) the committed steps of one streamline (all its halves)
    land in -- what the per-streamline-unique map counts once (R25)."""
    out = set()
    d0 = None
    for h in range(2 if getattr(w, "bidir", 0) else 1):
        _, _, _, d, vox = _half(w, seed_index, j, h, d0, 1)
        if h == 0:
            d0 = d
        out.update(vox)
    return out


def track_streamline(w, seed_index: int, j: int, max_points: int = 10**9):
    """All halves of one particle (two with ``w.bidir``): [(nsteps, reason, positions)]."""
    out = []
    d0 = None
    for h in range(2 if getattr(w, "bidir", 0) else 1):
        n, why, pos, d, _ = _half(w, seed_index, j, h, d0, max_points)
        if h == 0:
            d0 = d
        out.append((n, why, pos))
    return out


def _half(w, seed_index: int, j: int, half: int, d0, max_points: int):
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
    interp = getattr(w, "interp", 0)
    init_mode = getattr(w, "init_fibre", 0)

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
    d_first = None
    visited = []  # voxel of every committed step
    if vox is None or (half == 1 and d0 is None):
        return 0, 0, np.array(pos, np.float32), None, visited
    n = 0
    p = None if half == 0 else [-d0[a] for a in range(3)]
    while True:
        if n == w.max_steps:
            return n, 2, np.array(pos, np.float32), d_first, visited
        wd = philox4x32_10([n // 3, pid & _M, pid >> 32, half], key)
        s = (j % S) if getattr(w, "sample_mode", 0) == 1 else (wd[n % 3] * S) >> 32
        first = n == 0 and half == 0
        wi = None
        if interp or (first and init_mode):
            wi = philox4x32_10([n, pid & _M, pid >> 32, 2 + half], key)
        sv = vox
        if interp:
            u = _interp_voxel(q, wi, N, v.mask)
            if u is not None:
                sv = u
        vv = [[dy[jj, s, sv[0], sv[1], sv[2], a] for a in range(3)] for jj in range(F)]
        ff = [fr[jj, s, sv[0], sv[1], sv[2]] for jj in range(F)]
        if first:
            js = _first_fibre(init_mode, ff, fthr, wi[3] if wi is not None else 0)
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
                return n, 1, np.array(pos, np.float32), d_first, visited
            sg = np.float32(1.0) if dots[js] > np.float32(0) else np.float32(-1.0)
        d = [sg * vv[js][a] for a in range(3)]
        if first:
            d_first = d
        qn = [q[a] + h * d[a] for a in range(3)]
        vn = lookup(qn)
        if vn is None:
            return n, 0, np.array(pos, np.float32), d_first, visited
        q, p, vox = qn, d, vn
        n += 1
        visited.append(vn)
        if len(pos) < max_points:
            pos.append([q[a] + c[a] for a in range(3)])
