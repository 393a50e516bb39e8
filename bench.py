"""bench.py -- streamline steps/s of the B200 tracking hot path (BASELINE.json metric).

Default workload: BASELINE.json configs[2], the whole-brain-shaped phantom (128x128x70,
50 samples x 2 fibres, all WM seeds x 5000 particles, step 0.5, curvature 0.2, max 2000
steps), synthetic (phantom.whole_brain).  A "step" of this bench is one pass of the whole
hot path over that workload: pt_track (repacked records already resident, the persistent
tracking kernel, the map-sum overflow check) and, for N > 1, the NCCL reduce of the maps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config c3]

For N > 1 bench.py launches itself as N ranks (torch.distributed.run, one process per GPU,
NCCL) unless it already runs under torchrun; seeds are sharded in Z-order blocks with their
global ids and the maps are combined with one NCCL reduce.  Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "streamline steps/sec (and seeds/sec) at 1/2/4/8 B200; % of gather roofline"
CONFIG_TEXT = {
    "c3": "configs[2]: 128x128x70 whole-brain-shaped synthetic volume, 50 samples x 2 fibres, "
          "all WM seeds x 5000 particles, step 0.5 vox, curvature 0.2, max 2000 steps, fp32 records",
    "c4": "configs[3]: c3 with fp16 packed sample vectors (generator-rounded halves)",
    "c2": "configs[1]: 64x64x32 two-bundle 90deg crossing, 50 samples x 2 fibres, 1k seeds x 5000",
    "c2_dispersed": "configs[1] shape, dispersed (sigma 0.15, f jitter 0.03)",
    "c1": "configs[0]: 32x32x16 straight tube, 64 seeds x 1000",
    "c5": "configs[4]: HCP-scale 145x174x145, 50 samples x 3 fibres, fp16 records, all WM seeds x 10^4 "
          "particles (BASELINE quotes it on 8 B200; here per GPU)",
    "d1": "NEXT-1 paper mode: dataset-1-shaped 96x96x48, every brain voxel x 50 (one streamline per "
          "sample volume), step 0.1, dot threshold 0.9, MaxStep 1888 (Table II row 1 parameters)",
    "d2": "NEXT-1 paper mode: dataset-2-shaped 102x102x60, every brain voxel x 50, step 0.1, "
          "dot threshold 0.9, MaxStep 1888 (Table II row 4 parameters)",
}

MCMC_METRIC = "MCMC voxels/sec (Table III workload: 50 samples, L = 2, burn-in 500)"
MCMC_TEXT = {
    "m1": "NEXT-4 MCMC: dataset-1-shaped DWI 96x96x48, 205k valid voxels, 4 b0 + 60 dirs, N = 2, "
          "burn-in 500 + 50 samples x interval 2 (Table III row 1)",
    "m2": "NEXT-4 MCMC: dataset-2-shaped DWI 102x102x60, 402k valid voxels, 4 b0 + 60 dirs, N = 2, "
          "burn-in 500 + 50 samples x interval 2 (Table III row 2)",
    "m_small": "NEXT-4 MCMC: 24x24x16 brain, burn-in 100 + 10 samples x 2",
}
# Table III: valid voxels, CPU time, GPU time (HD 5870), context only
PAPER_TABLE3 = {"m1": {"voxels": 205082, "cpu_s": 1383, "gpu_s": 41.3, "speedup": 33.6},
                "m2": {"voxels": 402194, "cpu_s": 2724, "gpu_s": 80.1, "speedup": 34.0}}


def mcmc_flops_per_mh_step(n: int, N: int) -> int:
    """Algorithmic FP64 operations of one Metropolis-Hastings step: Eq. 1
    evaluated at the proposal for all n measurements, plus the Gaussian log-likelihood.
    Per measurement i: the ball term e^{-b_i d} (b_i d: 1 mul, exp: 1) weighted by (1 - sum
    f) (1 mul); per stick j: r_i . v_j (3 mul + 2 add), squared (1), times b_i d (1), exp (1),
    times f_j (1), added (1) = 10; the sum times S0 (1); the residual y_i - mu_i (1) and its
    square accumulated (1 mul + 1 add).  Per step: 1 - sum f (N adds) and the log posterior
    of M2/M3 (ln sigma, the 1/(2 sigma^2) scaling, the sin-theta priors and the
    accept test: 8).  exp and ln count as one operation each (the FP64 pipe spends ~20
    instructions on one -- the reason the measured fraction stays well below 1)."""
    return n * (3 + 10 * N + 1 + 3) + N + 8


def mcmc_flops_per_voxel_loop(n: int, N: int) -> int:
    """One loop = one MH step per parameter (NP = 3 + 3N, Fig. 2 / P:L147)."""
    return (3 + 3 * N) * mcmc_flops_per_mh_step(n, N)

# Table II of the paper, for context beside the NEXT-1 paper-mode workloads:
# (total fibre length = total steps, longest fibre) on the real CABI datasets, HD 5870.
PAPER_TABLE2 = {"d1": {"total_steps": 113822762, "longest": 453, "kernel_s": 3.02, "gpu_total_s": 6.74},
                "d2": {"total_steps": 305396623, "longest": 777, "kernel_s": 6.78, "gpu_total_s": 14.84}}


def _env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


# ----------------------------------------------------------------------------- clocks

class ClockSampler:
    """nvidia-smi sampling DURING the timed region (B200_PROFILING.md clocks line)."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except (OSError, ValueError):
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": max(mx), "samples": len(sm),
                "reasons": sorted(reasons)}


# ----------------------------------------------------------------------------- helpers

def _cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        return None


def _ncu_traffic(cfg, steps):
    """DRAM bytes (read + write) per launch of the tracking kernel from the committed ncu
    --set full capture (profiles/ncu_track_summary.json): bytes per committed step of that
    capture x this launch's steps (a capture may cover a seed subset, e.g. c5), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_track_summary.json")
    try:
        d = json.load(open(p))
        e = d.get("per_config", {}).get(cfg) or {}
        b = e.get("dram_bytes_per_step")
        return None if b is None else b * steps
    except (OSError, ValueError):
        return None


def _ncu_counters(cfg):
    """Counters of the committed ncu --set full capture of this config's tracking kernel
    (north star: achieved L2 / HBM sector throughput, warp execution efficiency), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_track_summary.json")
    try:
        e = json.load(open(p)).get("per_config", {}).get(cfg)
    except (OSError, ValueError):
        return None
    if not e:
        return None
    keys = ("tag", "warp_exec_efficiency", "issue_active_pct", "l1_hit_rate_pct", "l2_hit_rate_pct",
            "lts_throughput_pct", "l2_read_sectors_per_step", "l2_red_sectors_per_step", "dram_bytes_per_step",
            "warp_inst_per_32_steps")
    out = {k: e[k] for k in keys if k in e}
    out["source"] = "profiles/ncu_track_summary.json (ncu --set full capture, profiles/<tag>_" + cfg + "_track_ncu.md)"
    return out


def _workload(cfg):
    import phantom
    return phantom.config(cfg)


def _shard(w, rank, world):
    from paper_conf_ipps_xuzwrwxgxy12_b200 import sharding
    env = os.environ.get("PT_SHARD_BLOCK")  # experiments; 0 = seed i -> rank i mod N
    block = int(env) if env else None  # None: Z-order blocks of <= 1024 seeds (sharding.auto_block)
    seeds, ids = sharding.shard_seeds(w.seeds, w.seed_ids, rank, world, block=block)
    return w.replace(seeds=seeds, seed_ids=ids)


def _cpu_sample(w, target_s: float, threads: int):
    """Oracle sample of workload w: every k-th seed x ALL its particles (so the GPU can run
    the same pids through the bench's own launch and the two maps compare bit for bit),
    k sized from a calibration run so the sample takes ~target_s of wall time on `threads`
    host threads.  Returns (sample workload, particles per seed, every)."""
    import oracle
    import phantom
    cal = phantom.wm_seeds(w, every=max(1, w.nseeds // 64))
    t = time.perf_counter()
    r = oracle.track(cal, 0, 20, want_map=False)
    dt = time.perf_counter() - t
    rate1 = max(1.0, r["nsteps"].sum() / max(dt, 1e-6))          # steps/s on one core
    mean_len = max(1.0, float(r["nsteps"].mean()))
    particles = target_s * rate1 * threads / mean_len
    P = w.particles_per_seed
    nseeds = int(max(threads, min(w.nseeds, particles / P)))
    every = max(1, w.nseeds // nseeds)
    sub = phantom.wm_seeds(w, every=every)
    return sub, P, every


def _run_oracle_sample(sub, J, threads, keep=False, unique=False):
    import oracle
    t = time.perf_counter()
    r = oracle.track(sub, 0, J, want_map=True, threads=threads, want_unique=unique)
    dt = time.perf_counter() - t
    if keep:
        return int(r["nsteps"].sum()), dt, r
    return int(r["nsteps"].sum()), dt


# ----------------------------------------------------------------------------- reference arm

def run_reference(args):
    rank = _env_int("RANK", 0)
    if rank != 0:
        return 0
    import oracle
    oracle.build()
    w = _workload(args.config)
    threads = len(os.sched_getaffinity(0))
    sub, J, every = _cpu_sample(w, args.cpu_seconds, threads)
    for _ in range(args.warmup):
        _run_oracle_sample(sub, J, threads)
    steps = 0
    secs = 0.0
    for _ in range(args.steps):
        s, dt = _run_oracle_sample(sub, J, threads)
        steps += s
        secs += dt
    v = steps / secs
    desc = (f"{args.config}: every {every}th WM seed ({sub.nseeds} seeds) x all {J} particles; "
            f"oracle single-threaded per worker, {threads} worker threads")
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "steps/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": {"workload": CONFIG_TEXT.get(args.config, args.config),
                                        "sample": desc},
        "cpu_baseline": {"value": v, "unit": "steps/s", "cores": threads, "kind": "oracle",
                         "sample": desc},
        "e2e": {"value": v, "unit": "steps/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------------------- NEXT-4 MCMC arm

def _fp64_peak():
    """FP64 flop/s derived from the unit counts: 148 SMs x 64 FP64 lanes per SM per clock x
    2 (an FMA is two operations) x the measured max SM clock (MEASURED_PEAKS.json, else
    1965 MHz): 37.2 TFLOP/s at 1965 MHz."""
    p = _peaks()
    mhz = (p or {}).get("sm_max_mhz", 1965.0)
    return 148 * 64 * 2 * mhz * 1e6


def _mcmc_shard(d, rank, world):
    """Voxel v -> rank v mod N (results are keyed by the voxel index, so exact)."""
    from paper_conf_ipps_xuzwrwxgxy12_b200 import sharding
    if world == 1:
        return d
    return d.replace(mask=sharding.shard_voxels(d.mask, rank, world))


def run_mcmc(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_xuzwrwxgxy12_b200 as pt
    import phantom

    world = _env_int("WORLD_SIZE", 1)
    rank = _env_int("RANK", 0)
    local = _env_int("LOCAL_RANK", 0)
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    d = _mcmc_shard(phantom.mcmc_config(args.config), rank, world)
    tr = pt.Tracker(local)
    dd = d.replace(dwi=torch.as_tensor(d.dwi, device=dev), bvals=torch.as_tensor(d.bvals, device=dev),
                   bvecs=torch.as_tensor(d.bvecs, device=dev), mask=torch.as_tensor(d.mask, device=dev))
    NP = d.nparams
    out = torch.empty((NP, d.nsamples, d.nz, d.ny, d.nx), dtype=torch.float64, device=dev)
    for _ in range(args.warmup):
        tr.mcmc(dd, samples=out)
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    clocks.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    kms = []
    e0.record()
    for _ in range(args.steps):
        tr.mcmc(dd, samples=out)
        kms.append(tr.mcmc_stats()["kernel_ms"])
    e1.record()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ck = clocks.stop()
    ms = e0.elapsed_time(e1)
    st = tr.mcmc_stats()
    t = torch.tensor([ms, float(st["voxels"]), float(st["mh_steps"]), float(st["accepted"])],
                     dtype=torch.float64, device=dev)
    if world > 1:
        tm = t.clone()
        dist.all_reduce(tm, op=dist.ReduceOp.MAX)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        ms = float(tm[0])
    voxels, steps = float(t[1]), float(t[2])

    # e2e: host DWI in (pinned), host samples out (pinned), through the same C ABI call
    h = d.replace(dwi=torch.as_tensor(d.dwi).pin_memory(), bvals=torch.as_tensor(d.bvals),
                  bvecs=torch.as_tensor(d.bvecs), mask=torch.as_tensor(d.mask).pin_memory())
    out_h = torch.empty((NP, d.nsamples, d.nz, d.ny, d.nx), dtype=torch.float64).pin_memory()
    tr.mcmc(h, samples=out_h)
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    e2e_n = max(1, min(args.steps, 2))
    for _ in range(e2e_n):
        tr.mcmc(h, samples=out_h)
    e2e_s = (time.perf_counter() - t0) / e2e_n
    te = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)

    kmean = sum(kms) / len(kms)
    peak = _fp64_peak()
    ops = mcmc_flops_per_voxel_loop(int(d.nmeas), int(d.nfibres))
    ach = st["voxels"] * d.loops * ops / (kmean * 1e-3)
    roof = {"bound": "alu", "achieved": ach / 1e12, "peak": peak / 1e12,
            "unit": "TFLOP/s (FP64)", "frac": ach / peak, "traffic": None,
            "kernel_ms": kmean, "flops_per_voxel_loop": ops,
            "per_unit_source": "algorithmic: Eq. 1 (P:L67-69) at the proposal for all n measurements per MH "
                               "step, NP = 3 + 3N steps per loop (bench.mcmc_flops_per_mh_step; exp/ln = 1 op)",
            "peak_source": "derived: 148 SMs x 64 FP64 lanes x 2 (FMA) x sm_max_mhz"}
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        oracle.build()
        threads = len(os.sched_getaffinity(0))
        idx = np.flatnonzero(d.mask.ravel())
        cal = idx[:: max(1, idx.size // 16)][:16]
        t1 = time.perf_counter()
        oracle.mcmc(d, voxels=cal)
        per_vox = (time.perf_counter() - t1) / max(1, cal.size)
        nv = int(min(idx.size, max(threads, args.cpu_seconds * threads / max(per_vox, 1e-6))))
        pick = idx[:: max(1, idx.size // nv)]
        t1 = time.perf_counter()
        oracle.mcmc(d, voxels=pick, threads=threads)
        dt = time.perf_counter() - t1
        cpu = {"value": pick.size / dt, "unit": "voxels/s", "cores": threads, "kind": "oracle", "cpu_model": _cpu_model(),
               "sample": f"every {max(1, idx.size // nv)}th valid voxel ({pick.size} voxels) in {dt:.1f} s"}
    if rank == 0:
        line = {
            "metric": MCMC_METRIC, "value": voxels * args.steps / (ms * 1e-3), "unit": "voxels/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": MCMC_TEXT.get(args.config, args.config), "voxels": int(voxels),
                       "measurements": int(d.nmeas), "loops": d.loops, "parameters": NP,
                       "parallelism": f"voxel-sharded x{world}", "l2": "compute-bound (inputs read once per voxel)"},
            "mh_steps_per_s": steps * args.steps / (ms * 1e-3),
            "acceptance": float(t[3]) / max(1.0, steps),
            "paper_table3_context": PAPER_TABLE3.get(args.config),
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": {"value": voxels / float(te[0]), "unit": "voxels/s",
                    "h2d_bytes_per_step": int(d.dwi.nbytes + d.mask.nbytes + d.bvals.nbytes + d.bvecs.nbytes),
                    "d2h_bytes_per_step": int(out_h.numel() * 8)},
            "gpu_launches": 4 * args.steps,  # mask flags, cub select (2), mcmc_kernel
            "clocks": ck,
        }
        print(json.dumps(line), flush=True)
    tr.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_mcmc_reference(args):
    """Reference arm of the MCMC workload: the oracle on a bounded voxel sample."""
    import numpy as np
    import oracle
    import phantom
    if _env_int("RANK", 0) != 0:
        return 0
    oracle.build()
    d = phantom.mcmc_config(args.config)
    threads = len(os.sched_getaffinity(0))
    idx = np.flatnonzero(d.mask.ravel())
    cal = idx[:: max(1, idx.size // 16)][:16]
    t1 = time.perf_counter()
    oracle.mcmc(d, voxels=cal)
    per_vox = (time.perf_counter() - t1) / max(1, cal.size)
    nv = int(min(idx.size, max(threads, args.cpu_seconds / max(1, args.steps) * threads / max(per_vox, 1e-6))))
    pick = idx[:: max(1, idx.size // nv)]
    for _ in range(args.warmup):
        oracle.mcmc(d, voxels=pick[:threads], threads=threads)
    secs = 0.0
    for _ in range(args.steps):
        t1 = time.perf_counter()
        oracle.mcmc(d, voxels=pick, threads=threads)
        secs += time.perf_counter() - t1
    v = pick.size * args.steps / secs
    desc = f"{args.config}: every {max(1, idx.size // nv)}th valid voxel ({pick.size}); {threads} worker threads"
    print(json.dumps({
        "impl": "reference", "metric": MCMC_METRIC, "value": v, "unit": "voxels/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": {"workload": MCMC_TEXT.get(args.config, args.config), "sample": desc},
        "cpu_baseline": {"value": v, "unit": "voxels/s", "cores": threads, "kind": "oracle", "sample": desc},
        "e2e": {"value": v, "unit": "voxels/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}), flush=True)
    return 0


# ----------------------------------------------------------------------------- our arm

def run_ours(args):
    import hashlib

    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_xuzwrwxgxy12_b200 as pt
    from paper_conf_ipps_xuzwrwxgxy12_b200 import sharding

    world = _env_int("WORLD_SIZE", 1)
    rank = _env_int("RANK", 0)
    local = _env_int("LOCAL_RANK", 0)
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE {world} ranks (launch through "
                         "bench.py itself or torch.distributed.run with --nproc-per-node {args.gpus})")
    # BENCH_DIST_BACKEND=gloo + BENCH_SINGLE_DEVICE=1: test hook that runs the multi-rank
    # path with every rank on cuda:0 (NCCL cannot put two ranks on one GPU)
    backend = os.environ.get("BENCH_DIST_BACKEND", "nccl")
    if os.environ.get("BENCH_SINGLE_DEVICE") == "1":
        local = 0
    if world > 1:
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
        print(f"[bench rank {rank}/{world}] process group '{dist.get_backend()}' on cuda:{local} "
              f"({torch.cuda.get_device_name(local)}), nccl {torch.cuda.nccl.version()}",
              file=sys.stderr, flush=True)
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)

    w = _workload(args.config)
    if args.seed_every > 1:
        import phantom
        w = phantom.wm_seeds(w, every=args.seed_every)
    # NEXT-3 variants requested through --track-flags: the workload (and so the oracle of the
    # cpu_baseline / parity leg) carries the same semantics
    tf = args.track_flags
    w = w.replace(bidir=int(bool(tf & pt.PT_BIDIR)), interp=int(bool(tf & pt.PT_INTERP)),
                  init_fibre=1 if tf & pt.PT_INIT_RANDOM else (2 if tf & pt.PT_INIT_FWEIGHT else 0))
    unique = bool(tf & pt.PT_MAP_UNIQUE)
    mine = _shard(w, rank, world)
    tr = pt.Tracker(local)
    # load through the C ABI from pinned host memory: the paper's Copy3DImagesToGPU (P:L165,
    # "Transfer" in Table II), reported separately (load) and inside e2e_with_load
    vol = w.volume
    dy_h = torch.from_numpy(vol.dyads).pin_memory()
    f_h = torch.from_numpy(vol.f).pin_memory()
    m_h = torch.from_numpy(vol.mask).pin_memory()

    def load():
        tr.load_samples(dy_h, f_h, m_h, vol.nsamples, vol.nfibres)
        return tr.load_stats()

    load()
    ls = load()
    base_flags = args.track_flags | (pt.PT_SAMPLE_PER_STREAMLINE if getattr(w, "sample_mode", 0) else 0)
    if args.segments:
        tr.set_segments({"B": pt.SEGMENTS_B, "C": pt.SEGMENTS_C}.get(args.segments) or
                        [int(x) for x in args.segments.split(",")])
    V = vol.nx * vol.ny * vol.nz
    rb = pt.pt_record_bytes(vol.nfibres, pt.PT_F16 if vol.is_half else pt.PT_F32)
    seeds_d = torch.as_tensor(mine.seeds, device=dev).contiguous()
    ids_d = torch.as_tensor(mine.ids().astype(np.int64), device=dev).contiguous()
    out_map = torch.empty((vol.nz, vol.ny, vol.nx), dtype=torch.int32, device=dev)
    flush_buf = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)  # > L2 (126 MB)
    tparams = dict(step=w.step, curv_thr=w.curv_thr, fib_thr=w.fib_thr, max_steps=w.max_steps,
                   rng_seed=w.rng_seed, particles_per_seed=w.particles_per_seed)

    def one_step():
        flush_buf.fill_(1)  # evict L2 between steps
        tr.track(seeds_d, ids_d, out_map=out_map, flags=base_flags, want_map=not args.no_map, **tparams)
        if world > 1 and not args.no_map:
            sharding.reduce_map(out_map, dst=0)  # one NCCL reduce; int32 sum == uint32 sum

    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    kern_ms, track_ms = [], []
    e0.record()
    for _ in range(args.steps):
        one_step()
        if args.per_step_stats:
            s = tr.stats()
            kern_ms.append(s["kernel_ms"])
            track_ms.append(s["track_ms"])
    e1.record()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ck = clocks.stop()
    ms = e0.elapsed_time(e1)
    st = tr.stats()
    if not args.per_step_stats:
        kern_ms = [st["kernel_ms"]]
    my_steps = st["total_steps"]  # identical every step (deterministic)
    map_sha = None
    if rank == 0 and not args.no_map:
        mh = out_map.cpu().numpy().view(np.uint32)
        map_sha = hashlib.sha256(mh.tobytes()).hexdigest()
        if args.dump_map:
            np.save(args.dump_map, mh)
    t = torch.tensor([ms, float(my_steps), float(mine.nseeds), float(st["lane_active"]),
                      float(st["lane_slots"]), float(st["unique_visits"])], dtype=torch.float64, device=dev)

    def allreduce(x, op):
        # gloo (test hook) reduces host tensors
        if backend == "gloo" and x.is_cuda:
            h = x.cpu()
            dist.all_reduce(h, op=op)
            x.copy_(h)
        else:
            dist.all_reduce(x, op=op)

    if world > 1:
        tmax = t.clone()
        allreduce(tmax, dist.ReduceOp.MAX)
        allreduce(t, dist.ReduceOp.SUM)
        ms = float(tmax[0])
    total_steps = float(t[1])
    total_seeds = float(t[2])
    lane_frac = float(t[3] / t[4]) if float(t[4]) else None
    unique_visits = float(t[5])

    # ---- e2e through the C ABI with host buffers (pinned seeds in, pinned map out), and the
    # same with the sample-volume load (pinned host volumes -> H2D + repack) in every step
    seeds_h = torch.as_tensor(mine.seeds).pin_memory()
    ids_h = torch.as_tensor(mine.ids().astype(np.int64)).pin_memory()
    map_h = torch.empty((vol.nz, vol.ny, vol.nx), dtype=torch.int32).pin_memory()
    e2e_steps = max(1, min(args.steps, 3))

    def e2e_step(with_load):
        flush_buf.fill_(1)
        if with_load:
            load()
        tr.track(seeds_h, ids_h, out_map=map_h, flags=base_flags, **tparams)
        if world > 1:
            # the host map is reduced over the process group as the step's result
            mt = map_h.to(dev, non_blocking=True)
            sharding.reduce_map(mt, dst=0)
            if rank == 0:
                map_h.copy_(mt)

    e2e_vals = {False: None, True: None}
    if not args.no_e2e:
        e2e_step(False)  # warm
    for with_load in (() if args.no_e2e else (False, True)):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step(with_load)
        torch.cuda.synchronize()
        te = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        if world > 1:
            allreduce(te, dist.ReduceOp.MAX)
        e2e_vals[with_load] = total_steps * e2e_steps / float(te[0])

    # ---- roofline (dominant kernel = the tracking kernel)
    kms = sum(kern_ms) / len(kern_ms)
    # SURVEY §8(d) algorithmic bytes per committed step: one record read + one 4-B map
    # atomic (counted as its 4 B, as §8(d) lists it); per seed 12 B of seed + 8 B of id
    alg_bytes = my_steps * (rb + 4) + mine.nseeds * (12 + 8)
    achieved = alg_bytes / (kms * 1e-3) / 1e9
    peaks = _peaks()
    peak = peaks["hbm_gbs"] if peaks else 6650.0
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak,
            "traffic": _ncu_traffic(args.config, my_steps) if not args.track_flags else None,
            "peak_source": "measured (MEASURED_PEAKS.json hbm_gbs)" if peaks else "fallback 6.65 TB/s",
            "bytes_per_step": rb + 4, "kernel_ms": kms,
            "kernel_ms_steps": kern_ms, "track_ms_steps": track_ms}
    gather = None
    if rank == 0 and not args.no_gather_bench:
        rec_bytes_total = V * vol.nsamples * rb
        r_hbm = tr.gather_bench(int(rec_bytes_total), rb)
        r_l2 = tr.gather_bench(64 * 1024 * 1024, rb)
        sec_per_step = max(1, rb // 32)
        sps = my_steps / (kms * 1e-3)
        gather = {"r_gather_hbm_sectors_per_s": r_hbm, "r_gather_l2_sectors_per_s": r_l2,
                  "hbm_copy_sectors_per_s": peak * 1e9 / 32,
                  "frac_of_r_gather_hbm": sps * sec_per_step / r_hbm,
                  "frac_of_r_gather_l2": sps * sec_per_step / r_l2,
                  "frac_of_hbm_copy_sectors": sps * sec_per_step / (peak * 1e9 / 32),
                  "sectors_per_step": sec_per_step}

    cpu = None
    parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        oracle.build()
        threads = len(os.sched_getaffinity(0))
        sub, J, every = _cpu_sample(w, args.cpu_seconds, threads)
        s, dt, r = _run_oracle_sample(sub, J, threads, keep=True, unique=unique)
        cpu = {"value": s / dt, "unit": "steps/s", "cores": threads, "kind": "oracle", "cpu_model": _cpu_model(),
               "sample": f"every {every}th WM seed ({sub.nseeds} seeds) x all {J} particles: "
                         f"{s} steps in {dt:.1f} s"}
        if not args.no_parity:
            # the same pids through the bench's own launch (flags as timed: no per-particle
            # outputs) -> map; and through the outputs instantiation -> per-streamline results
            sd = torch.as_tensor(sub.seeds, device=dev).contiguous()
            si = torch.as_tensor(sub.ids().astype(np.int64), device=dev).contiguous()
            gm = tr.track(sd, si, flags=base_flags, **tparams)
            torch.cuda.synchronize()
            gmap = gm.cpu().numpy().view(np.uint32).astype(np.uint64)
            rmap = r["umap"] if unique else r["map"]  # PT_MAP_UNIQUE: streamlines per voxel (R25)
            rec = pt.PT_REC_LEN | pt.PT_REC_REASON | pt.PT_REC_END
            tr.track(sd, si, flags=base_flags | rec, want_map=False, **tparams)
            torch.cuda.synchronize()
            g = tr.get_paths()
            div = ((g["nsteps"].astype(np.int64) != r["nsteps"]) | (g["reason"] != r["reason"]) |
                   np.any(g["end"].view(np.uint32) != r["end"].view(np.uint32), axis=1))
            l1 = float(np.abs(gmap.astype(np.int64) - rmap.astype(np.int64)).sum()) / max(1, int(rmap.sum()))
            parity = {"sample": cpu["sample"], "streamlines": int(div.size), "divergent": int(div.sum()),
                      "divergent_fraction": float(div.mean()), "map_l1_rel": l1,
                      "map_bit_exact": bool(np.array_equal(gmap, rmap)),
                      "kernel": "map: the timed launch (flags as benched); per-streamline: the outputs instantiation",
                      "bar": "divergent <= 1e-4, map L1 rel <= 1e-4 (north_star); expected 0 / 0"}

    emulated = None
    if rank == 0 and world == 1 and args.emulate_ranks:
        # Projected multi-GPU scaling on ONE GPU: each rank's shard of an N-way split is
        # timed back to back; N GPUs would finish when the slowest shard does, plus one NCCL
        # reduce of the map (not timed here).  Context only: SCALE runs measure the real thing.
        emulated = {}
        for N in args.emulate_ranks:
            times, steps_r = [], []
            for r_ in range(N):
                sub_ = _shard(w, r_, N)
                sd = torch.as_tensor(sub_.seeds, device=dev).contiguous()
                si = torch.as_tensor(sub_.ids().astype(np.int64), device=dev).contiguous()
                for it in range(2):  # warm-up + timed
                    flush_buf.fill_(1)
                    tr.track(sd, si, out_map=out_map, flags=base_flags, **tparams)
                    st_r = tr.stats()
                times.append(st_r["track_ms"])
                steps_r.append(st_r["total_steps"])
            emulated[str(N)] = {"shard_ms": times, "shard_steps": steps_r,
                                "projected_value": sum(steps_r) / (max(times) * 1e-3),
                                "imbalance_max_over_mean": max(times) / (sum(times) / len(times))}
        torch.cuda.synchronize()

    lengths = None
    if rank == 0 and not args.no_lengths and not (base_flags & pt.PT_MAP_UNIQUE):
        # one more (untimed) pass with per-particle lengths: the Eq. 4 / Fig. 5 statistics
        tr.track(seeds_d, ids_d, out_map=out_map, flags=base_flags | pt.PT_REC_LEN, **tparams)
        torch.cuda.synchronize()
        ns = tr.get_paths(nsteps=True, reason=False, end=False, on_device=True)["nsteps"]
        hist = torch.zeros(65536, dtype=torch.int64, device=dev)
        for c0 in range(0, ns.numel(), 1 << 27):
            hist += torch.bincount(ns[c0:c0 + (1 << 27)].to(torch.int32) & 0xFFFF, minlength=65536)
        h = hist.cpu().numpy()
        nz = np.nonzero(h)[0]
        tot = int((h * np.arange(65536)).sum())
        cnt = int(h.sum())
        mean = tot / max(1, cnt)
        # semilog fit of the length histogram between the 5th and 95th percentiles (Fig. 5c)
        cdf = np.cumsum(h) / max(1, cnt)
        lo, hi = int(np.searchsorted(cdf, 0.05)), int(np.searchsorted(cdf, 0.95))
        xs = np.arange(max(lo, 1), max(hi, lo + 2))
        ys = h[xs]
        keep = ys > 0
        slope = float(np.polyfit(xs[keep], np.log(ys[keep]), 1)[0]) if keep.sum() > 2 else None
        lengths = {"streamlines": cnt, "total_steps": tot, "mean": mean,
                   "longest": int(nz.max()) if nz.size else 0,
                   "lambda_mle": 1.0 / mean if mean > 0 else None,
                   "lambda_semilog_fit": -slope if slope is not None else None,
                   "fit_range": [int(xs[0]), int(xs[-1])],
                   "context": "Eq. 4 / Fig. 5 (P:L229-249): exponential fibre-length law"}
        if args.config in PAPER_TABLE2:
            lengths["paper_table2_context"] = PAPER_TABLE2[args.config]

    if rank == 0:
        value = total_steps * args.steps / (ms * 1e-3)
        line = {
            "metric": METRIC, "value": value, "unit": "steps/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f32", "data": "synthetic",
            "config": {"workload": CONFIG_TEXT.get(args.config, args.config),
                       "seeds": int(total_seeds), "particles_per_seed": w.particles_per_seed,
                       "particles": int(total_seeds) * w.particles_per_seed,
                       "steps_per_pass": int(total_steps),
                       "mean_steps_per_streamline": total_steps / max(1.0, total_seeds * w.particles_per_seed),
                       "record_bytes": rb, "records": "fp16" if vol.is_half else "fp32",
                       "record_layout": "bricks of %d^3 voxels" % (1 << int(os.environ.get("PT_BRICK", "4")))
                                        if int(os.environ.get("PT_BRICK", "4")) else "raster",
                       "track_flags": base_flags,
                       "parallelism": f"seed-sharded x{world}" + (" + NCCL reduce" if world > 1 else ""),
                       "l2": "inputs > L2 (record volume %.2f GB) and a 256 MiB L2 flush between steps"
                             % (V * vol.nsamples * rb / 1e9)},
            "seeds_per_s": total_seeds * args.steps / (ms * 1e-3),
            "active_lane_fraction": lane_frac,
            "steps_per_lane_iteration": (my_steps / st["lane_active"]) if st["lane_active"] else None,
            "unique_visits_per_pass": int(unique_visits) if (base_flags & pt.PT_MAP_UNIQUE) else None,
            "parity": parity,
            "map_sha256": map_sha,
            "lengths": lengths,
            "load": {"h2d_ms": ls["h2d_ms"], "repack_ms": ls["repack_ms"], "h2d_bytes": ls["h2d_bytes"],
                     "record_bytes": ls["record_bytes"],
                     "h2d_gb_per_s": ls["h2d_bytes"] / max(1e-9, ls["h2d_ms"] * 1e-3) / 1e9,
                     "what": "pt_load_samples from pinned host volumes: the paper's Copy3DImagesToGPU "
                             "(P:L165, Table II 'Transfer'), per GPU, untimed in value"},
            "emulated_scaling": emulated,
            "roofline": roof,
            "gather_roofline": gather,
            "ncu": _ncu_counters(args.config) if not args.track_flags else None,
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_vals[False], "unit": "steps/s",
                    "h2d_bytes_per_step": int(seeds_h.numel() * 4 + ids_h.numel() * 8),
                    "d2h_bytes_per_step": int(map_h.numel() * 4)},
            "e2e_with_load": {"value": e2e_vals[True], "unit": "steps/s",
                              "h2d_bytes_per_step": int(seeds_h.numel() * 4 + ids_h.numel() * 8 + ls["h2d_bytes"]),
                              "d2h_bytes_per_step": int(map_h.numel() * 4)},
            # per pt_track: seed_keys, cub radix sort (histogram, exclusive sum, 4 onesweep
            # passes), the tracking kernel, map_sum -- the ncu launch list
            # (profiles/r02b_c3_launches.md); the L2 flush is torch's fill kernel, not counted
            "gpu_launches": 9 * args.steps,
            "clocks": ck,
        }
        print(json.dumps(line), flush=True)
    tr.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def _self_launch(args, argv):
    """bench.py --gpus N with N > 1 and no torch.distributed environment: re-launch this
    script as N ranks (torch.distributed.run, one process per GPU, NCCL), with NCCL's
    communicator initialisation log on stderr so the rank count is visible."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    env.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes", "1", "--nproc-per-node", str(args.gpus),
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *argv]
    print("bench.py: launching " + " ".join(cmd), file=sys.stderr, flush=True)
    return subprocess.call(cmd, env=env)


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c3")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-gather-bench", action="store_true")
    ap.add_argument("--no-per-step-stats", dest="per_step_stats", action="store_false")
    ap.add_argument("--no-map", action="store_true", help="diagnostic: no visitation map")
    ap.add_argument("--emulate-ranks", type=lambda x: [int(v) for v in x.split(",") if v], default=[],
                    help="e.g. 2,4,8: time each rank's seed shard back to back on one GPU and "
                         "report the projected N-GPU throughput (max shard time)")
    ap.add_argument("--no-lengths", action="store_true",
                    help="skip the streamline-length statistics (untimed extra pass with PT_REC_LEN)")
    ap.add_argument("--no-parity", action="store_true",
                    help="skip the GPU run of the cpu_baseline sample (the parity report)")
    ap.add_argument("--no-e2e", action="store_true", help="experiments: skip the e2e legs")
    ap.add_argument("--dump-map", default="", help="rank 0 saves the (reduced) map of the last step (.npy)")
    ap.add_argument("--tag", default="", help="free-form label echoed by experiment scripts")
    ap.add_argument("--seed-every", type=int, default=1,
                    help="diagnostic (profiling only): every k-th seed of the workload")
    ap.add_argument("--track-flags", type=int, default=0,
                    help="extra pt_params.flags for ablations (e.g. 256 = PT_KERNEL_SIMPLE, "
                         "512 = PT_SEED_ORDER_INPUT)")
    ap.add_argument("--segments", default="",
                    help="schedule of the PT_KERNEL_SEGMENTED ablation (--track-flags 65536): "
                         "B, C or a comma list of intervals (the paper's NumIteration[])")
    argv = sys.argv[1:] if argv is None else list(argv)
    args = ap.parse_args(argv)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return _self_launch(args, argv)
    if args.warmup < 3 and args.impl == "ours" and not os.environ.get("BENCH_ALLOW_FEW_WARMUP"):
        args.warmup = 3
    if args.config.startswith("m"):
        if args.impl == "reference":
            return run_mcmc_reference(args)
        return run_mcmc(args)
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
