"""Oracle loader -- TEST INFRASTRUCTURE ONLY.

ctypes binding of ``oracle/oracle.c``, the plain single-threaded CPU reference of the
tracking hot path (see oracle.h for the contract and citations).  Only ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py`` (cpu_baseline leg, ``--impl reference``) may
import this module.  It imports nothing from the CUDA package and the CUDA package
imports nothing from here.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_SRC_MCMC = os.path.join(_HERE, "oracle_mcmc.c")
_HDR = os.path.join(_HERE, "oracle.h")
_LIB = os.environ.get("ORACLE_LIB") or os.path.join(_HERE, "liboracle.so")  # ORACLE_LIB: sanitizer build
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
          "-Wall", "-Wextra"]
SANITIZE = ["-fsanitize=address,undefined", "-fno-sanitize-recover=all", "-fno-omit-frame-pointer", "-g"]

END_MASK, END_CURV, END_MAXLEN = 0, 1, 2


def build(force: bool = False, out: Optional[str] = None, sanitize: bool = False) -> str:
    """Compile liboracle.so with gcc (no FMA contraction, no fast-math).  ``sanitize``: an
    ASan + UBSan build (load it with LD_PRELOAD=libasan.so and ORACLE_LIB=<out>)."""
    lib_path = out or _LIB
    srcs = [_SRC, _SRC_MCMC]
    stale = (not os.path.exists(lib_path) or
             os.path.getmtime(lib_path) < max(os.path.getmtime(f) for f in srcs + [_HDR]))
    if force or stale:
        tmp = lib_path + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, *(SANITIZE if sanitize else []), "-o", tmp, *srcs, "-lm"])
        os.replace(tmp, lib_path)
    return lib_path


class _Volume(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
                ("nsamples", ctypes.c_int32), ("nfibres", ctypes.c_int32),
                ("is_half", ctypes.c_int32), ("dyads", ctypes.c_void_p),
                ("f", ctypes.c_void_p), ("mask", ctypes.c_void_p)]


class _Params(ctypes.Structure):
    _fields_ = [("step", ctypes.c_float), ("curv_thr", ctypes.c_float),
                ("fib_thr", ctypes.c_float), ("max_steps", ctypes.c_int32),
                ("rng_seed", ctypes.c_uint64), ("particles_per_seed", ctypes.c_int64),
                ("sample_mode", ctypes.c_int32), ("bidir", ctypes.c_int32),
                ("interp", ctypes.c_int32), ("init_fibre", ctypes.c_int32)]


class _Dwi(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
                ("nmeas", ctypes.c_int32), ("dwi", ctypes.c_void_p), ("bvals", ctypes.c_void_p),
                ("bvecs", ctypes.c_void_p), ("mask", ctypes.c_void_p)]


class _McmcParams(ctypes.Structure):
    _fields_ = [("nfibres", ctypes.c_int32), ("burnin", ctypes.c_int32),
                ("nsamples", ctypes.c_int32), ("interval", ctypes.c_int32),
                ("adapt_every", ctypes.c_int32), ("rng_seed", ctypes.c_uint64),
                ("fixed", ctypes.c_uint32)]


_lib = None
_lock = threading.Lock()


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = ctypes.CDLL(_LIB if os.environ.get("ORACLE_LIB") else build())
            vp = ctypes.c_void_p
            L.oracle_philox4x32_10.argtypes = [vp, vp, vp]
            L.oracle_half_to_float.argtypes = [ctypes.c_uint16]
            L.oracle_half_to_float.restype = ctypes.c_float
            L.oracle_half_to_float_array.argtypes = [vp, vp, ctypes.c_int64]
            L.oracle_axis_index.argtypes = [ctypes.c_float, ctypes.c_int32]
            L.oracle_axis_index.restype = ctypes.c_int64
            L.oracle_sample_index.argtypes = [ctypes.c_uint32, ctypes.c_uint32]
            L.oracle_sample_index.restype = ctypes.c_uint32
            L.oracle_track.argtypes = [ctypes.POINTER(_Volume), ctypes.POINTER(_Params), vp, vp,
                                       ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                                       vp, vp, vp, vp, vp, ctypes.c_int32, vp, ctypes.c_int32, vp, vp]
            L.oracle_track.restype = ctypes.c_int
            L.oracle_mcmc_signal.argtypes = [ctypes.c_int, vp, ctypes.c_int, vp, vp, vp]
            L.oracle_mcmc_signal.restype = None
            L.oracle_mcmc_draw.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                                           ctypes.c_uint32, vp, vp]
            L.oracle_mcmc_draw.restype = None
            L.oracle_mcmc.argtypes = [ctypes.POINTER(_Dwi), ctypes.POINTER(_McmcParams), vp,
                                      ctypes.c_int64, ctypes.c_int64, vp, vp]
            L.oracle_mcmc.restype = ctypes.c_int
            _lib = L
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data


# ----------------------------------------------------------------------------- primitives

def philox(ctr, key) -> np.ndarray:
    c = np.ascontiguousarray(ctr, np.uint32)
    k = np.ascontiguousarray(key, np.uint32)
    out = np.zeros(4, np.uint32)
    lib().oracle_philox4x32_10(c.ctypes.data, k.ctypes.data, out.ctypes.data)
    return out


def half_to_float(bits: np.ndarray) -> np.ndarray:
    b = np.ascontiguousarray(bits, np.uint16)
    out = np.empty(b.shape, np.float32)
    lib().oracle_half_to_float_array(b.ctypes.data, out.ctypes.data, b.size)
    return out


def axis_index(q: float, n_axis: int) -> int:
    return int(lib().oracle_axis_index(ctypes.c_float(q), n_axis))


def sample_index(w: int, nsamples: int) -> int:
    return int(lib().oracle_sample_index(w, nsamples))


# ----------------------------------------------------------------------------- tracking

def _structs(volume, step, curv_thr, fib_thr, max_steps, rng_seed, P, sample_mode=0, bidir=0,
             interp=0, init_fibre=0):
    v = volume
    vs = _Volume(v.nx, v.ny, v.nz, v.nsamples, v.nfibres, 1 if v.dyads.dtype == np.float16 else 0,
                 v.dyads.ctypes.data, v.f.ctypes.data, v.mask.ctypes.data)
    ps = _Params(step, curv_thr, fib_thr, max_steps, rng_seed, P, sample_mode, bidir, interp,
                 init_fibre)
    return vs, ps


def track(w, j_begin: int = 0, j_end: Optional[int] = None, *, want_map: bool = True,
          want_particles: bool = True, path_stride: int = 0, threads: int = 1,
          labels: Optional[np.ndarray] = None, ntargets: int = 0, want_unique: bool = False) -> dict:
    """Run the oracle on workload ``w`` (a phantom.Workload or duck-typed equivalent).

    Returns dict(map=uint64[Z][Y][X] or None, nsteps=int32[n], reason=uint8[n],
    end=float32[n][3], paths=float32[n][path_stride][3] or None, conn=uint64[nseeds][ntargets]
    or None, umap=uint64[Z][Y][X] streamlines per voxel (R25) with ``want_unique`` else None),
    particles ordered (seed index, j) -- with ``w.bidir`` two entries per particle
    (seed index, j, half), n = 2 * nseeds * npp.  ``threads`` > 1 runs independent single-threaded oracle calls on
    disjoint seed shards (seed i -> worker i mod threads) and sums their maps.
    """
    v = w.volume
    P = int(w.particles_per_seed)
    j_end = P if j_end is None else int(j_end)
    npp = j_end - j_begin
    seeds = np.ascontiguousarray(w.seeds, np.float32)
    ids = np.ascontiguousarray(w.ids(), np.uint64)
    ns = seeds.shape[0]
    bidir = int(getattr(w, "bidir", 0))
    H = 2 if bidir else 1                          # entries per particle
    n = ns * npp * H
    vs, ps = _structs(v, w.step, w.curv_thr, w.fib_thr, w.max_steps, w.rng_seed, P,
                      int(getattr(w, "sample_mode", 0)), bidir, int(getattr(w, "interp", 0)),
                      int(getattr(w, "init_fibre", 0)))
    nsteps = np.zeros(n, np.int32) if want_particles else None
    reason = np.zeros(n, np.uint8) if want_particles else None
    end = np.zeros((n, 3), np.float32) if want_particles else None
    paths = np.zeros((n, path_stride, 3), np.float32) if path_stride > 0 else None
    L = lib()
    threads = max(1, min(int(threads), ns)) if ns else 1

    lab = None if labels is None else np.ascontiguousarray(labels, np.uint8)
    T = int(ntargets) if lab is not None else 0

    def run(shard: np.ndarray, mp: Optional[np.ndarray], um: Optional[np.ndarray]):
        sd = np.ascontiguousarray(seeds[shard])
        si = np.ascontiguousarray(ids[shard])
        m = len(shard) * npp * H
        ln = np.zeros(m, np.int32) if want_particles else None
        lr = np.zeros(m, np.uint8) if want_particles else None
        le = np.zeros((m, 3), np.float32) if want_particles else None
        lp = np.zeros((m, path_stride, 3), np.float32) if paths is not None else None
        lc = np.zeros((len(shard), T), np.uint64) if T else None
        rc = L.oracle_track(ctypes.byref(vs), ctypes.byref(ps), sd.ctypes.data, si.ctypes.data,
                            len(shard), j_begin, j_end, _ptr(mp), _ptr(ln), _ptr(lr), _ptr(le),
                            _ptr(lp), path_stride, _ptr(lab), T, _ptr(lc), _ptr(um))
        if rc != 0:
            raise ValueError(f"oracle_track rejected its arguments (rc={rc})")
        return ln, lr, le, lp, lc

    maps = [np.zeros((v.nz, v.ny, v.nx), np.uint64) if want_map else None for _ in range(threads)]
    umaps = [np.zeros((v.nz, v.ny, v.nx), np.uint64) if want_unique else None for _ in range(threads)]
    shards = [np.arange(t, ns, threads) for t in range(threads)]
    results = [None] * threads
    if threads == 1:
        results[0] = run(shards[0], maps[0], umaps[0])
    else:
        def worker(t):
            results[t] = run(shards[t], maps[t], umaps[t])
        th = [threading.Thread(target=worker, args=(t,)) for t in range(threads)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        if any(r is None for r in results):
            raise RuntimeError("oracle worker failed")
    conn = np.zeros((ns, T), np.uint64) if T else None
    for t, shard in enumerate(shards):
        ln, lr, le, lp, lc = results[t]
        if conn is not None and len(shard):
            conn[shard] = lc
        if len(shard) == 0:
            continue
        rows = (shard[:, None] * (npp * H) + np.arange(npp * H)[None, :]).ravel()
        if want_particles:
            nsteps[rows] = ln
            reason[rows] = lr
            end[rows] = le
        if paths is not None:
            paths[rows] = lp
    mp = None
    if want_map:
        mp = maps[0]
        for m in maps[1:]:
            mp += m
    um = None
    if want_unique:
        um = umaps[0]
        for m in umaps[1:]:
            um += m
    return dict(map=mp, nsteps=nsteps, reason=reason, end=end, paths=paths, conn=conn, umap=um)


# ----------------------------------------------------------------------------- NEXT-4 MCMC

def mcmc_signal(nfibres: int, omega, bvals, bvecs) -> np.ndarray:
    """Eq. 1 for one parameter vector (S0, d, sigma, f1, th1, ph1, ...)."""
    om = np.ascontiguousarray(omega, np.float64)
    b = np.ascontiguousarray(bvals, np.float32)
    r = np.ascontiguousarray(bvecs, np.float32)
    mu = np.zeros(b.size, np.float64)
    lib().oracle_mcmc_signal(int(nfibres), om.ctypes.data, b.size, b.ctypes.data, r.ctypes.data,
                             mu.ctypes.data)
    return mu


def mcmc_draw(seed: int, loop: int, voxel: int, k: int):
    """(z, log u) of MH step (loop, voxel, k) (M6)."""
    z = np.zeros(1, np.float64)
    lu = np.zeros(1, np.float64)
    lib().oracle_mcmc_draw(seed, loop, voxel, k, z.ctypes.data, lu.ctypes.data)
    return float(z[0]), float(lu[0])


def mcmc(d, *, init: Optional[np.ndarray] = None, fixed: int = 0, threads: int = 1,
         voxels: Optional[np.ndarray] = None) -> dict:
    """Run the MCMC oracle on a phantom.DwiWorkload ``d``.

    Returns dict(samples=float64 [NP][S][Z][Y][X] (0 outside the sampled voxels),
    accepted=uint32 [NP][Z][Y][X]).  ``voxels`` (sorted linear indices) restricts the run to
    a subset of the mask; ``threads`` > 1 runs independent single-threaded oracle calls on
    disjoint voxel ranges.
    """
    NP = 3 + 3 * int(d.nfibres)
    V = d.nx * d.ny * d.nz
    dwi = np.ascontiguousarray(d.dwi, np.float32)
    bv = np.ascontiguousarray(d.bvals, np.float32)
    bc = np.ascontiguousarray(d.bvecs, np.float32)
    mask = np.ascontiguousarray(d.mask, np.uint8)
    if voxels is not None:
        sub = np.zeros(V, np.uint8)
        sub[np.asarray(voxels, np.int64)] = 1
        mask = (sub.reshape(mask.shape) & (mask != 0)).astype(np.uint8)
    ds = _Dwi(d.nx, d.ny, d.nz, bv.size, dwi.ctypes.data, bv.ctypes.data, bc.ctypes.data,
              mask.ctypes.data)
    ps = _McmcParams(int(d.nfibres), int(d.burnin), int(d.nsamples), int(d.interval),
                     int(d.adapt_every), int(d.rng_seed), int(fixed))
    ini = None if init is None else np.ascontiguousarray(init, np.float64).reshape(NP, V)
    samples = np.zeros((NP, int(d.nsamples), V), np.float64)
    acc = np.zeros((NP, V), np.uint32)
    L = lib()
    flat = np.flatnonzero(mask.ravel())
    threads = max(1, min(int(threads), max(1, flat.size)))
    cuts = [0] + [int(flat[(flat.size * t) // threads]) for t in range(1, threads)] + [V]
    errs = []

    def run(t):
        rc = L.oracle_mcmc(ctypes.byref(ds), ctypes.byref(ps), _ptr(ini), cuts[t], cuts[t + 1],
                           samples.ctypes.data, acc.ctypes.data)
        if rc != 0:
            errs.append(rc)

    if threads == 1:
        run(0)
    else:
        th = [threading.Thread(target=run, args=(t,)) for t in range(threads)]
        for t in th:
            t.start()
        for t in th:
            t.join()
    if errs:
        raise ValueError(f"oracle_mcmc rejected its arguments (rc={errs[0]})")
    return dict(samples=samples.reshape(NP, int(d.nsamples), d.nz, d.ny, d.nx),
                accepted=acc.reshape(NP, d.nz, d.ny, d.nx))
