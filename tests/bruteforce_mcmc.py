"""Third, independent MCMC sampler (NEXT-4) for tiny chains: pure Python floats (binary64)
with the ``math`` module, Python-int Philox (tests/bruteforce.py).  Shares nothing with
``oracle/`` or the CUDA path; it restates DESIGN.md §12 (M1-M9) directly:

  Eq. 1  mu_i = S0 [(1 - sum f) e^{-b d} + sum_j f_j e^{-b d (r.v_j)^2}]
  log posterior     -(n+1) log sigma - SSE / (2 sigma^2) + sum_j log|sin theta_j|
  MH step k         omega'_k = omega_k + prop_k z, accept iff log u < lp' - lp
  adaptation        every K loops prop_k *= sqrt(5 (acc_k + 1) / (3 (rej_k + 1)))
  samples           after loop t >= burnin with (t - burnin + 1) % L == 0
"""
from __future__ import annotations

import math

from tests.bruteforce import philox4x32_10

TAG = 0x4D434D43


def draw(seed, loop, voxel, k):
    w = philox4x32_10([loop, voxel, k, TAG], [seed & 0xFFFFFFFF, seed >> 32])
    u1 = (w[0] + 0.5) / 2.0 ** 32
    u2 = w[1] / 2.0 ** 32
    u3 = (w[2] + 0.5) / 2.0 ** 32
    return math.sqrt(-2.0 * math.log(u1)) * math.cos(6.283185307179586 * u2), math.log(u3)


def signal(N, w, bvals, bvecs):
    sumf = 0.0
    for j in range(N):
        sumf += w[3 + 3 * j]
    out = []
    for b, r in zip(bvals, bvecs):
        b = float(b)
        rx, ry, rz = (float(c) for c in r)
        bd = b * w[1]
        acc = (1.0 - sumf) * math.exp(-bd)
        for j in range(N):
            th, ph = w[4 + 3 * j], w[5 + 3 * j]
            vx, vy, vz = math.sin(th) * math.cos(ph), math.sin(th) * math.sin(ph), math.cos(th)
            dot = (rx * vx + ry * vy) + rz * vz
            acc += w[3 + 3 * j] * math.exp(-(bd * (dot * dot)))
        out.append(w[0] * acc)
    return out


def log_post(N, w, y, bvals, bvecs):
    mu = signal(N, w, bvals, bvecs)
    sse = 0.0
    for yi, mi in zip(y, mu):
        sse += (yi - mi) * (yi - mi)
    lp = -(len(y) + 1) * math.log(w[2]) - sse / (2.0 * w[2] * w[2])
    for j in range(N):
        s = abs(math.sin(w[4 + 3 * j]))
        lp += math.log(s) if s > 0 else -math.inf
    return lp


def support(N, w):
    if not (w[0] > 0 and w[1] > 0 and w[2] > 0):
        return False
    fs = [w[3 + 3 * j] for j in range(N)]
    if not all(f >= 0 for f in fs):
        return False
    t = 0.0
    for f in fs:
        t += f
    return t <= 1.0


def chain(d, voxel, init, fixed=0):
    """Run one voxel's chain from ``init`` (list of NP floats); returns the samples
    [S][NP] and the accepted counts [NP]."""
    N = d.nfibres
    NP = 3 + 3 * N
    V = d.nx * d.ny * d.nz
    y = [float(d.dwi.reshape(-1, V)[i, voxel]) for i in range(d.nmeas)]
    w = [float(x) for x in init]
    prop = [0.01 * w[0], 0.1 * w[1], 0.1 * w[2]] + [0.05, 0.1, 0.1] * N
    acc = [0] * NP
    rej = [0] * NP
    tot = [0] * NP
    lp = log_post(N, w, y, d.bvals, d.bvecs)
    out = []
    for t in range(d.burnin + d.nsamples * d.interval):
        for k in range(NP):
            if fixed >> k & 1:
                continue
            z, lu = draw(d.rng_seed, t, voxel, k)
            wn = list(w)
            wn[k] = w[k] + prop[k] * z
            if not support(N, wn):
                rej[k] += 1
                continue
            lpn = log_post(N, wn, y, d.bvals, d.bvecs)
            if lu < lpn - lp:
                w, lp = wn, lpn
                acc[k] += 1
                tot[k] += 1
            else:
                rej[k] += 1
        if (t + 1) % d.adapt_every == 0:
            for k in range(NP):
                prop[k] *= math.sqrt((5.0 * (acc[k] + 1)) / (3.0 * (rej[k] + 1)))
                acc[k] = rej[k] = 0
        if t >= d.burnin and (t - d.burnin + 1) % d.interval == 0:
            out.append(list(w))
    return out, tot
