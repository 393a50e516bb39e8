"""B200-native probabilistic-streamlining particle stepper (Xu et al., IPDPSW 2012).

Thin Python binding of the C ABI in ``include/pt.h`` (``libpt.so``, sm_100a).  Every
function here only marshals arguments: the whole hot path (repack, stepping, counting)
runs in the CUDA kernels of ``csrc/``.  There is no CPU fallback: importing the binding
without a built ``libpt.so`` raises, and every call without a CUDA device fails with the
library's own error.  PyTorch supplies device memory and streams only.

Low-level names mirror the C ABI (``pt_create``, ``pt_load_samples``, ``pt_track``,
``pt_get_paths``, ``pt_get_stats``, ``pt_gather_bench``...); ``Tracker`` is the same
calls with torch tensors.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

from ._build import LIB, build  # noqa: F401

__all__ = [
    "PtError", "lib", "Tracker", "pt_create", "pt_destroy", "pt_last_error", "pt_set_stream",
    "pt_load_samples", "pt_track", "pt_get_paths", "pt_get_stats", "pt_gather_bench",
    "pt_record_bytes", "PT_F32", "PT_F16", "PT_REC_LEN", "PT_REC_REASON", "PT_REC_END",
    "PT_REC_PATHS", "PT_MAP_ACCUMULATE", "PT_KERNEL_SIMPLE", "PT_SEED_ORDER_INPUT",
    "PT_SAMPLE_PER_STREAMLINE", "PT_REC_CONN", "PT_BIDIR", "PT_INTERP", "PT_INIT_RANDOM",
    "PT_INIT_FWEIGHT", "PT_KERNEL_VARIANT", "variant_flags", "pt_mcmc", "pt_get_mcmc_stats",
    "pt_mcmc_to_volume", "pt_dwi_shape", "pt_mcmc_params", "PT_KERNEL_SEGMENTED", "pt_set_segments",
    "PT_MAP_UNIQUE", "SEGMENTS_B", "SEGMENTS_C", "pt_load_targets", "pt_get_connectivity", "PT_END_MASK",
    "PT_END_CURV", "PT_END_MAXLEN", "pt_get_load_stats", "pt_rng_draws", "EXPORTS",
]

PT_OK, PT_ERR_ARG, PT_ERR_STATE, PT_ERR_OOM, PT_ERR_CUDA, PT_ERR_OVERFLOW = range(6)
PT_F32, PT_F16 = 0, 1
PT_END_MASK, PT_END_CURV, PT_END_MAXLEN = 0, 1, 2
PT_REC_LEN = 1 << 0
PT_REC_REASON = 1 << 1
PT_REC_END = 1 << 2
PT_REC_PATHS = 1 << 3
PT_MAP_ACCUMULATE = 1 << 4
PT_REC_CONN = 1 << 5
PT_KERNEL_SIMPLE = 1 << 8
PT_SEED_ORDER_INPUT = 1 << 9
PT_SAMPLE_PER_STREAMLINE = 1 << 10
PT_BIDIR = 1 << 11
PT_INTERP = 1 << 12
PT_INIT_RANDOM = 1 << 13
PT_INIT_FWEIGHT = 1 << 14
PT_KERNEL_VARIANT = 1 << 15
PT_KERNEL_SEGMENTED = 1 << 16
PT_MAP_UNIQUE = 1 << 18  # NEXT-2: per-streamline-unique visitation map (R25)
# the paper's increasing-interval segmentation strategies
SEGMENTS_B = (1, 2, 5, 10, 20, 50, 100, 200, 500)
SEGMENTS_C = (1, 1, 2, 2, 5, 5, 10, 10, 20, 20, 50, 50, 100, 100, 200, 200)


def variant_flags(bidir: int = 0, interp: int = 0, init_fibre: int = 0) -> int:
    """pt_params.flags bits of the NEXT-3 variants (R22-R24)."""
    return ((PT_BIDIR if bidir else 0) | (PT_INTERP if interp else 0) |
            {0: 0, 1: PT_INIT_RANDOM, 2: PT_INIT_FWEIGHT}[int(init_fibre)])

# every symbol include/pt.h declares
EXPORTS = ["pt_create", "pt_destroy", "pt_last_error", "pt_set_stream", "pt_load_samples",
           "pt_track", "pt_get_paths", "pt_get_stats", "pt_gather_bench", "pt_record_bytes",
           "pt_load_targets", "pt_get_connectivity", "pt_mcmc", "pt_get_mcmc_stats",
           "pt_mcmc_to_volume", "pt_set_segments", "pt_get_load_stats", "pt_rng_draws"]

_STATUS = {1: "PT_ERR_ARG", 2: "PT_ERR_STATE", 3: "PT_ERR_OOM", 4: "PT_ERR_CUDA", 5: "PT_ERR_OVERFLOW"}


class PtError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class pt_volume(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
                ("nsamples", ctypes.c_int32), ("nfibres", ctypes.c_int32), ("dtype", ctypes.c_int32)]


class pt_params(ctypes.Structure):
    _fields_ = [("step", ctypes.c_float), ("curv_thr", ctypes.c_float), ("fib_thr", ctypes.c_float),
                ("max_steps", ctypes.c_int32), ("rng_seed", ctypes.c_uint64),
                ("particles_per_seed", ctypes.c_int64), ("flags", ctypes.c_uint32),
                ("path_stride", ctypes.c_int32)]


class pt_paths(ctypes.Structure):
    _fields_ = [("nsteps", ctypes.c_void_p), ("reason", ctypes.c_void_p), ("end_xyz", ctypes.c_void_p),
                ("paths", ctypes.c_void_p), ("capacity", ctypes.c_int64), ("count", ctypes.c_int64),
                ("path_stride", ctypes.c_int32)]


class pt_stats(ctypes.Structure):
    _fields_ = [("total_steps", ctypes.c_uint64), ("particles", ctypes.c_uint64),
                ("lane_active", ctypes.c_uint64), ("lane_slots", ctypes.c_uint64),
                ("map_sum", ctypes.c_uint64), ("overflow", ctypes.c_int32),
                ("kernel_ms", ctypes.c_float), ("track_ms", ctypes.c_float),
                ("unique_visits", ctypes.c_uint64)]


class pt_load_stats(ctypes.Structure):
    _fields_ = [("h2d_ms", ctypes.c_float), ("repack_ms", ctypes.c_float), ("h2d_bytes", ctypes.c_uint64),
                ("record_bytes", ctypes.c_uint64)]


class pt_dwi_shape(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
                ("nmeas", ctypes.c_int32)]


class pt_mcmc_params(ctypes.Structure):
    _fields_ = [("nfibres", ctypes.c_int32), ("burnin", ctypes.c_int32), ("nsamples", ctypes.c_int32),
                ("interval", ctypes.c_int32), ("adapt_every", ctypes.c_int32),
                ("rng_seed", ctypes.c_uint64), ("fixed", ctypes.c_uint32)]


class pt_mcmc_stats(ctypes.Structure):
    _fields_ = [("voxels", ctypes.c_uint64), ("mh_steps", ctypes.c_uint64), ("accepted", ctypes.c_uint64),
                ("kernel_ms", ctypes.c_float)]


_lib = None


def lib() -> ctypes.CDLL:
    """Load the in-tree libpt.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB):
        raise ImportError(f"{LIB} is missing: run __graft_entry__.build() (nvcc, sm_100a); "
                          "this package has no CPU fallback")
    L = ctypes.CDLL(LIB)
    vp, P = ctypes.c_void_p, ctypes.POINTER
    L.pt_create.argtypes = [ctypes.c_int, P(vp)]
    L.pt_create.restype = ctypes.c_int
    L.pt_destroy.argtypes = [vp]
    L.pt_destroy.restype = None
    L.pt_last_error.argtypes = [vp]
    L.pt_last_error.restype = ctypes.c_char_p
    L.pt_set_stream.argtypes = [vp, vp]
    L.pt_set_stream.restype = ctypes.c_int
    L.pt_load_samples.argtypes = [vp, P(pt_volume), vp, vp, vp]
    L.pt_load_samples.restype = ctypes.c_int
    L.pt_track.argtypes = [vp, vp, vp, ctypes.c_int64, P(pt_params), vp]
    L.pt_track.restype = ctypes.c_int
    L.pt_get_paths.argtypes = [vp, P(pt_paths)]
    L.pt_get_paths.restype = ctypes.c_int
    L.pt_get_stats.argtypes = [vp, P(pt_stats)]
    L.pt_get_stats.restype = ctypes.c_int
    L.pt_gather_bench.argtypes = [vp, ctypes.c_int64, ctypes.c_int32, P(ctypes.c_double)]
    L.pt_gather_bench.restype = ctypes.c_int
    L.pt_load_targets.argtypes = [vp, vp, ctypes.c_int32]
    L.pt_load_targets.restype = ctypes.c_int
    L.pt_get_connectivity.argtypes = [vp, vp, ctypes.c_int64, P(ctypes.c_int64)]
    L.pt_get_connectivity.restype = ctypes.c_int
    L.pt_mcmc.argtypes = [vp, P(pt_dwi_shape), vp, vp, vp, vp, P(pt_mcmc_params), vp, vp, vp]
    L.pt_mcmc.restype = ctypes.c_int
    L.pt_get_mcmc_stats.argtypes = [vp, P(pt_mcmc_stats)]
    L.pt_get_mcmc_stats.restype = ctypes.c_int
    L.pt_mcmc_to_volume.argtypes = [vp, P(pt_dwi_shape), ctypes.c_int32, ctypes.c_int32, vp, vp, vp, vp]
    L.pt_mcmc_to_volume.restype = ctypes.c_int
    L.pt_set_segments.argtypes = [vp, vp, ctypes.c_int32]
    L.pt_set_segments.restype = ctypes.c_int
    L.pt_get_load_stats.argtypes = [vp, P(pt_load_stats)]
    L.pt_get_load_stats.restype = ctypes.c_int
    L.pt_rng_draws.argtypes = [vp, vp, vp, vp, ctypes.c_int64, ctypes.c_uint64, ctypes.c_uint32, vp, vp,
                               P(ctypes.c_int64)]
    L.pt_rng_draws.restype = ctypes.c_int
    L.pt_record_bytes.argtypes = [ctypes.c_int32, ctypes.c_int32]
    L.pt_record_bytes.restype = ctypes.c_int32
    _lib = L
    return L


def _check(ctx, rc: int):
    if rc != PT_OK:
        msg = lib().pt_last_error(ctx)
        raise PtError(rc, (msg or b"").decode(errors="replace"))


# ------------------------------------------------------------------ C-ABI names (marshalling)

def pt_create(device: int = 0) -> int:
    h = ctypes.c_void_p()
    _check(None, lib().pt_create(device, ctypes.byref(h)))
    return h.value


def pt_destroy(ctx) -> None:
    lib().pt_destroy(ctx)


def pt_last_error(ctx) -> str:
    return (lib().pt_last_error(ctx) or b"").decode(errors="replace")


def pt_set_stream(ctx, stream: int) -> None:
    _check(ctx, lib().pt_set_stream(ctx, stream))


def pt_record_bytes(nfibres: int, dtype: int) -> int:
    return int(lib().pt_record_bytes(nfibres, dtype))


def pt_load_samples(ctx, nx, ny, nz, nsamples, nfibres, dtype, dyads_ptr, f_ptr, mask_ptr) -> None:
    v = pt_volume(nx, ny, nz, nsamples, nfibres, dtype)
    _check(ctx, lib().pt_load_samples(ctx, ctypes.byref(v), dyads_ptr, f_ptr, mask_ptr))


def pt_track(ctx, seeds_ptr, ids_ptr, nseeds: int, params: pt_params, map_ptr) -> None:
    _check(ctx, lib().pt_track(ctx, seeds_ptr, ids_ptr, nseeds, ctypes.byref(params), map_ptr))


def pt_get_paths(ctx, out: pt_paths) -> pt_paths:
    _check(ctx, lib().pt_get_paths(ctx, ctypes.byref(out)))
    return out


def pt_get_stats(ctx) -> pt_stats:
    s = pt_stats()
    _check(ctx, lib().pt_get_stats(ctx, ctypes.byref(s)))
    return s


def pt_load_targets(ctx, labels_ptr, ntargets: int) -> None:
    _check(ctx, lib().pt_load_targets(ctx, labels_ptr, ntargets))


def pt_get_connectivity(ctx, out_ptr, capacity: int) -> int:
    n = ctypes.c_int64()
    _check(ctx, lib().pt_get_connectivity(ctx, out_ptr, capacity, ctypes.byref(n)))
    return n.value


def pt_mcmc(ctx, shape: pt_dwi_shape, dwi_ptr, bvals_ptr, bvecs_ptr, mask_ptr, params: pt_mcmc_params,
            init_ptr, samples_ptr, accepted_ptr) -> None:
    _check(ctx, lib().pt_mcmc(ctx, ctypes.byref(shape), dwi_ptr, bvals_ptr, bvecs_ptr, mask_ptr,
                              ctypes.byref(params), init_ptr, samples_ptr, accepted_ptr))


def pt_get_mcmc_stats(ctx) -> pt_mcmc_stats:
    s = pt_mcmc_stats()
    _check(ctx, lib().pt_get_mcmc_stats(ctx, ctypes.byref(s)))
    return s


def pt_mcmc_to_volume(ctx, shape: pt_dwi_shape, nfibres: int, nsamples: int, samples_ptr, mask_ptr,
                      dyads_ptr, f_ptr) -> None:
    _check(ctx, lib().pt_mcmc_to_volume(ctx, ctypes.byref(shape), nfibres, nsamples, samples_ptr,
                                        mask_ptr, dyads_ptr, f_ptr))


def pt_set_segments(ctx, intervals) -> None:
    arr = (ctypes.c_int32 * len(intervals))(*[int(x) for x in intervals])
    _check(ctx, lib().pt_set_segments(ctx, arr, len(intervals)))


def pt_get_load_stats(ctx) -> pt_load_stats:
    s = pt_load_stats()
    _check(ctx, lib().pt_get_load_stats(ctx, ctypes.byref(s)))
    return s


def pt_rng_draws(ctx, pid_ptr, block_ptr, stream_ptr, n: int, rng_seed: int, nsamples: int, words_ptr,
                 samples_ptr) -> int:
    mm = ctypes.c_int64()
    _check(ctx, lib().pt_rng_draws(ctx, pid_ptr, block_ptr, stream_ptr, n, rng_seed, nsamples, words_ptr,
                                   samples_ptr, ctypes.byref(mm)))
    return mm.value


def pt_gather_bench(ctx, buffer_bytes: int, record_bytes: int) -> float:
    r = ctypes.c_double()
    _check(ctx, lib().pt_gather_bench(ctx, buffer_bytes, record_bytes, ctypes.byref(r)))
    return r.value


# ------------------------------------------------------------------ torch convenience

def _ptr(a) -> Optional[int]:
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        if not a.flags.c_contiguous:
            raise ValueError("array must be C-contiguous")
        return a.ctypes.data
    if not a.is_contiguous():
        raise ValueError("tensor must be contiguous")
    return a.data_ptr()


def _contig(a):
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return np.ascontiguousarray(a)
    return a.contiguous()


def _dt(a) -> str:
    """dtype name of a numpy array or torch tensor ('float32', 'uint8', ...)."""
    return str(a.dtype).replace("torch.", "")


def _expect(name: str, a, dtypes, shape=None) -> None:
    """Argument check before a pointer crosses the ABI: the C side reads raw bytes, so a
    wrong dtype or shape would be silent garbage or an out-of-bounds read."""
    if _dt(a) not in dtypes:
        raise TypeError(f"{name}: dtype {_dt(a)}, expected one of {sorted(dtypes)}")
    if shape is not None:
        got = tuple(int(d) for d in a.shape)
        if len(got) != len(shape) or any(e is not None and g != e for g, e in zip(got, shape)):
            raise ValueError(f"{name}: shape {got}, expected {tuple('*' if e is None else e for e in shape)}")


class Tracker:
    """One context on one GPU; tensors in, tensors out (torch supplies memory/streams)."""

    def __init__(self, device: int = 0):
        import torch
        self.torch = torch
        self.device = torch.device("cuda", device)
        self.ctx = pt_create(device)
        self.shape = None

    def close(self):
        if self.ctx:
            pt_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _stream(self):
        pt_set_stream(self.ctx, self.torch.cuda.current_stream(self.device).cuda_stream)

    def load_samples(self, dyads, f, mask, nsamples: int, nfibres: int) -> None:
        """dyads [F][S][Z][Y][X][3], f [F][S][Z][Y][X] (float32 or float16), mask [Z][Y][X]
        uint8; numpy (host) or torch (host or cuda) arrays."""
        half = _dt(dyads) == "float16"
        _expect("mask", mask, {"uint8", "bool"}, (None, None, None))
        nz, ny, nx = (int(d) for d in mask.shape)
        _expect("dyads", dyads, {"float32", "float16"}, (nfibres, nsamples, nz, ny, nx, 3))
        _expect("f", f, {_dt(dyads)}, (nfibres, nsamples, nz, ny, nx))
        self._stream()
        pt_load_samples(self.ctx, nx, ny, nz, nsamples, nfibres, PT_F16 if half else PT_F32,
                        _ptr(dyads), _ptr(f), _ptr(mask))
        self.shape = (nz, ny, nx)

    def load_volume(self, vol) -> None:
        """A phantom.Volume-like object (dyads, f, mask, nsamples, nfibres)."""
        self.load_samples(vol.dyads, vol.f, vol.mask, vol.nsamples, vol.nfibres)

    def track(self, seeds, seed_ids=None, *, step: float, curv_thr: float, fib_thr: float,
              max_steps: int, rng_seed: int, particles_per_seed: int, flags: int = 0,
              path_stride: int = 0, out_map=None, want_map: bool = True):
        """Enqueue pt_track on the current torch stream; returns the map (a cuda int32
        tensor [Z][Y][X] holding the uint32 counts bit for bit, unless ``out_map`` is
        given) or None."""
        torch = self.torch
        if want_map and out_map is None and self.shape is not None:
            out_map = torch.empty(self.shape, dtype=torch.int32, device=self.device)
        prm = pt_params(step, curv_thr, fib_thr, max_steps, rng_seed, particles_per_seed, flags,
                        path_stride)
        seeds, seed_ids = _contig(seeds), _contig(seed_ids)
        _expect("seeds", seeds, {"float32"}, (None, 3))
        n = int(seeds.shape[0])
        if seed_ids is not None:
            _expect("seed_ids", seed_ids, {"uint64", "int64"}, (n,))
        if want_map and out_map is not None:
            _expect("out_map", out_map, {"int32", "uint32"}, self.shape)
        self._stream()
        pt_track(self.ctx, _ptr(seeds), _ptr(seed_ids), n, prm, _ptr(out_map) if want_map else None)
        return out_map if want_map else None

    def track_workload(self, w, flags: int = 0, path_stride: int = 0, seeds=None, seed_ids=None,
                       out_map=None, want_map: bool = True):
        if getattr(w, "sample_mode", 0) == 1:
            flags |= PT_SAMPLE_PER_STREAMLINE
        flags |= variant_flags(getattr(w, "bidir", 0), getattr(w, "interp", 0),
                               getattr(w, "init_fibre", 0))
        seeds = w.seeds if seeds is None else seeds
        if seed_ids is None and w.seed_ids is not None:
            seed_ids = w.seed_ids
        return self.track(seeds, seed_ids, step=w.step, curv_thr=w.curv_thr, fib_thr=w.fib_thr,
                          max_steps=w.max_steps, rng_seed=w.rng_seed,
                          particles_per_seed=w.particles_per_seed, flags=flags,
                          path_stride=path_stride, out_map=out_map, want_map=want_map)

    def stats(self) -> dict:
        s = pt_get_stats(self.ctx)
        return {k: getattr(s, k) for k, _ in pt_stats._fields_}

    def get_paths(self, nsteps=True, reason=True, end=True, paths=False, on_device=False) -> dict:
        """Per-particle outputs of the last track: host numpy arrays, or cuda tensors with
        ``on_device`` (nsteps as int16 holding the uint16 bits, reason as uint8)."""
        q = pt_get_paths(self.ctx, pt_paths())
        n, stride = q.count, q.path_stride
        out = {}
        bufs = pt_paths()
        bufs.capacity = n
        torch = self.torch

        def alloc(name, shape, npdt, tdt):
            a = torch.empty(shape, dtype=tdt, device=self.device) if on_device else np.empty(shape, npdt)
            out[name] = a
            return _ptr(a)
        if nsteps:
            bufs.nsteps = alloc("nsteps", (n,), np.uint16, torch.int16)
        if reason:
            bufs.reason = alloc("reason", (n,), np.uint8, torch.uint8)
        if end:
            bufs.end_xyz = alloc("end", (n, 3), np.float32, torch.float32)
        if paths:
            bufs.paths = alloc("paths", (n, stride, 3), np.float32, torch.float32)
        pt_get_paths(self.ctx, bufs)
        return out

    def load_targets(self, labels, ntargets: int) -> None:
        """Target regions for the seed x target matrix (uint8 [Z][Y][X], 0 = none, t+1)."""
        labels = _contig(labels)
        if labels is not None:
            _expect("labels", labels, {"uint8"}, self.shape)
        self._stream()
        pt_load_targets(self.ctx, _ptr(labels), ntargets)

    def connectivity(self) -> np.ndarray:
        """Seed x target matrix (uint32 [nseeds][ntargets]) of the last PT_REC_CONN track."""
        n = pt_get_connectivity(self.ctx, None, 0)
        out = np.empty(n, np.uint32)
        pt_get_connectivity(self.ctx, out.ctypes.data, n)
        return out

    def set_segments(self, intervals) -> None:
        """Schedule of the PT_KERNEL_SEGMENTED ablation (the paper's NumIteration[])."""
        pt_set_segments(self.ctx, intervals)

    def load_stats(self) -> dict:
        """Timing of the last load_samples: H2D copy and repack (device ms), bytes."""
        s = pt_get_load_stats(self.ctx)
        return {k: getattr(s, k) for k, _ in pt_load_stats._fields_}

    def rng_draws(self, pid, block, stream, rng_seed: int, nsamples: int):
        """Device self-test of the tracking RNG (pt_rng_draws): returns (words uint32 [n][4],
        sample indices uint32 [n][3], blocks that differ from curand_Philox4x32_10)."""
        pid = np.ascontiguousarray(pid, np.uint64)
        block = np.ascontiguousarray(block, np.uint32)
        stream = np.ascontiguousarray(stream, np.uint32)
        n = pid.size
        if block.size != n or stream.size != n:
            raise ValueError("pid, block and stream must have the same length")
        words = np.zeros((n, 4), np.uint32)
        samples = np.zeros((n, 3), np.uint32)
        self._stream()
        mm = pt_rng_draws(self.ctx, pid.ctypes.data, block.ctypes.data, stream.ctypes.data, n, rng_seed,
                          nsamples, words.ctypes.data, samples.ctypes.data)
        return words, samples, mm

    def gather_bench(self, buffer_bytes: int, record_bytes: int) -> float:
        self._stream()
        return pt_gather_bench(self.ctx, buffer_bytes, record_bytes)

    # ------------------------------------------------------------------ NEXT-4 MCMC

    def mcmc(self, d, *, init=None, fixed: int = 0, accepted: bool = False, samples=None):
        """pt_mcmc on a phantom.DwiWorkload-like ``d`` (dwi [n][Z][Y][X] float32, bvals,
        bvecs, mask, nfibres, burnin, nsamples, interval, adapt_every, rng_seed).  Inputs
        may be numpy (host) or torch tensors; returns (samples, accepted): a cuda float64
        tensor [NP][S][Z][Y][X] (or the given ``samples`` buffer) and a cuda int32 tensor
        [NP][Z][Y][X] holding the uint32 counts, or None."""
        torch = self.torch
        NP = 3 + 3 * int(d.nfibres)
        nz, ny, nx = d.mask.shape
        shape = pt_dwi_shape(nx, ny, nz, int(np.asarray(d.bvals).size if isinstance(d.bvals, np.ndarray)
                                                else d.bvals.numel()))
        prm = pt_mcmc_params(int(d.nfibres), int(d.burnin), int(d.nsamples), int(d.interval),
                             int(d.adapt_every), int(d.rng_seed), int(fixed))
        if samples is None:
            samples = torch.empty((NP, int(d.nsamples), nz, ny, nx), dtype=torch.float64, device=self.device)
        acc = torch.empty((NP, nz, ny, nx), dtype=torch.int32, device=self.device) if accepted else None
        dwi, bv, bc, mask = (_contig(x) for x in (d.dwi, d.bvals, d.bvecs, d.mask))
        nm = int(shape.nmeas)
        _expect("dwi", dwi, {"float32"}, (nm, nz, ny, nx))
        _expect("bvals", bv, {"float32"}, (nm,))
        _expect("bvecs", bc, {"float32"}, (nm, 3))
        _expect("mask", mask, {"uint8", "bool"}, (nz, ny, nx))
        if samples is not None:
            _expect("samples", samples, {"float64"}, (NP, int(d.nsamples), nz, ny, nx))
        ini = _contig(init)
        if ini is not None:
            _expect("init", ini, {"float64"}, (NP, nz, ny, nx))
        self._stream()
        pt_mcmc(self.ctx, shape, _ptr(dwi), _ptr(bv), _ptr(bc), _ptr(mask), prm, _ptr(ini),
                _ptr(samples), _ptr(acc))
        return samples, acc

    def mcmc_stats(self) -> dict:
        s = pt_get_mcmc_stats(self.ctx)
        return {k: getattr(s, k) for k, _ in pt_mcmc_stats._fields_}

    def mcmc_to_volume(self, samples, mask, nfibres: int):
        """Sample volumes for load_samples from pt_mcmc samples (R20 conversion on the GPU):
        returns (dyads [N][S][Z][Y][X][3], f [N][S][Z][Y][X]) float32 cuda tensors."""
        torch = self.torch
        S = int(samples.shape[1])
        nz, ny, nx = mask.shape
        dy = torch.empty((nfibres, S, nz, ny, nx, 3), dtype=torch.float32, device=self.device)
        f = torch.empty((nfibres, S, nz, ny, nx), dtype=torch.float32, device=self.device)
        mask = _contig(mask)
        self._stream()
        pt_mcmc_to_volume(self.ctx, pt_dwi_shape(nx, ny, nz, 1), nfibres, S, _ptr(samples), _ptr(mask),
                          _ptr(dy), _ptr(f))
        return dy, f
