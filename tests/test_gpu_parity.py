"""GPU <-> oracle parity through the C ABI (``-m gpu``; needs a B200 and libpt.so).

Bar (BASELINE.json north_star): per-streamline (nsteps, reason, end
point bits) and the uint32 visitation maps bit-exact vs the oracle on identical generated
inputs.  Every comparison below is exact; the tolerance the north star allows (<= 1e-4
divergent streamlines, map L1 relative difference <= 1e-4) is asserted as a fallback
report only where a full-size run is sampled.
"""
from __future__ import annotations

import os

import numpy as np
import pytest

import oracle
import phantom

pytestmark = pytest.mark.gpu

REC_ALL = None  # set in fixture


@pytest.fixture(scope="module")
def pt():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_ipps_xuzwrwxgxy12_b200 as m
    m.build()
    global REC_ALL
    REC_ALL = m.PT_REC_LEN | m.PT_REC_REASON | m.PT_REC_END
    return m


@pytest.fixture(scope="module")
def tracker(pt):
    t = pt.Tracker(0)
    yield t
    t.close()


def _threads():
    return max(1, len(os.sched_getaffinity(0)))


def gpu_run(tr, w, flags=None, path_stride=0, **kw):
    import torch
    flags = REC_ALL if flags is None else flags
    tr.load_volume(w.volume)
    m = tr.track_workload(w, flags=flags, path_stride=path_stride, **kw)
    torch.cuda.synchronize()
    out = tr.get_paths(nsteps=bool(flags & 1), reason=bool(flags & 2), end=bool(flags & 4),
                       paths=bool(flags & 8))
    out["map"] = None if m is None else m.cpu().numpy().view(np.uint32)
    out["stats"] = tr.stats()
    return out


def paths_equal(a, b):
    """Bit-identical points; unused points are NaN on both sides (payload may differ)."""
    na, nb = np.isnan(a), np.isnan(b)
    return np.array_equal(na, nb) and np.array_equal(a[~na].view(np.uint32), b[~nb].view(np.uint32))


def assert_parity(g, r, idx=None, check_map=True):
    sl = slice(None) if idx is None else idx
    assert np.array_equal(g["nsteps"][sl].astype(np.int64), r["nsteps"].astype(np.int64)), \
        f"nsteps: {np.count_nonzero(g['nsteps'][sl].astype(np.int64) != r['nsteps'])} differ"
    assert np.array_equal(g["reason"][sl], r["reason"])
    assert np.array_equal(g["end"][sl].view(np.uint32), r["end"].view(np.uint32))
    if check_map:
        assert np.array_equal(g["map"].astype(np.uint64), r["map"])


# ----------------------------------------------------------------------------- full configs

@pytest.mark.parametrize("simple", [False, True])
def test_c1_full(pt, tracker, simple):
    """BASELINE configs[0]: every particle and the full map, both kernels."""
    w = phantom.config("c1")
    g = gpu_run(tracker, w, REC_ALL | (pt.PT_KERNEL_SIMPLE if simple else 0))
    r = oracle.track(w)
    assert_parity(g, r)
    assert g["stats"]["total_steps"] == int(r["nsteps"].sum())


def test_c2_full(pt, tracker):
    """BASELINE configs[1] (zero dispersion): 1000 seeds x 5000 particles, all of them."""
    w = phantom.config("c2")
    g = gpu_run(tracker, w)
    r = oracle.track(w, threads=_threads())
    assert_parity(g, r)


def test_c2_dispersed_full(pt, tracker):
    """configs[1] shape, dispersed (sigma 0.15, f jitter 0.03): the full map and every
    particle's (nsteps, reason, end)."""
    w = phantom.config("c2_dispersed")
    g = gpu_run(tracker, w)
    r = oracle.track(w, threads=_threads())
    assert_parity(g, r)
    assert g["stats"]["total_steps"] == int(r["nsteps"].sum()) == int(g["map"].sum(dtype=np.uint64))


# ----------------------------------------------------------------------------- paths

@pytest.mark.parametrize("half", [False, True])
@pytest.mark.parametrize("F", [1, 2, 3])
def test_paths_bit_identical(pt, tracker, F, half):
    """Per-step positions bit-identical on small brain-shaped volumes (F = 1..3, fp32 and
    fp16 records), with a ragged particle count (P = 37, not a multiple of the chunk)."""
    w = phantom.whole_brain(nx=40, ny=36, nz=24, semi=(17.0, 15.0, 10.0), nsamples=16, nfibres=F,
                            particles_per_seed=37)
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 150))
    if half:
        w = phantom.to_half(w)
    stride = 512
    g = gpu_run(tracker, w, REC_ALL | pt.PT_REC_PATHS, path_stride=stride)
    r = oracle.track(w, path_stride=stride, threads=_threads())
    assert_parity(g, r)
    assert paths_equal(g["paths"], r["paths"])


@pytest.mark.parametrize("simple", [False, True])
def test_crossing_dispersed_paths(pt, tracker, simple):
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=60, particles_per_seed=40, nsamples=50)
    g = gpu_run(tracker, w, REC_ALL | pt.PT_REC_PATHS | (pt.PT_KERNEL_SIMPLE if simple else 0),
                path_stride=300)
    r = oracle.track(w, path_stride=300)
    assert_parity(g, r)
    assert paths_equal(g["paths"], r["paths"])


# ----------------------------------------------------------------------------- record layout

@pytest.mark.parametrize("brick", [0, 4])
def test_record_layout_bricks(pt, tracker, brick, monkeypatch):
    """The bricked record layout (PT_BRICK = log2 brick edge) changes where a
    record lives, never which record a step reads: on a volume whose dims are multiples of
    no brick edge (41 x 37 x 23, so every brick row / column / slab is ragged) the main
    kernel, the no-refill kernel and the variant kernel stay bit-exact with the oracle."""
    import torch
    monkeypatch.setenv("PT_BRICK", str(brick))
    w = phantom.whole_brain(nx=41, ny=37, nz=23, semi=(18.0, 16.0, 10.0), nsamples=12, nfibres=2,
                            particles_per_seed=33)
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 120))
    r = oracle.track(w, threads=_threads())
    for extra in (0, pt.PT_KERNEL_SIMPLE, pt.PT_KERNEL_VARIANT):
        g = gpu_run(tracker, w, REC_ALL | extra)
        assert_parity(g, r)
    # a variant that reads other voxels than the nearest one (probabilistic interpolation)
    wb = phantom.whole_brain(nx=41, ny=37, nz=23, semi=(18.0, 16.0, 10.0), nsamples=12, nfibres=2,
                             particles_per_seed=9)
    wb = phantom.wm_seeds(wb, every=max(1, wb.nseeds // 60)).replace(bidir=1, interp=1)
    gi = gpu_run(tracker, wb)
    ri = oracle.track(wb, threads=_threads())
    assert_parity(gi, ri)
    torch.cuda.synchronize()


def test_record_layout_rejects_other_bricks(pt, monkeypatch):
    """Only the two compiled layouts are accepted (PT_ERR_ARG otherwise, nothing loaded)."""
    monkeypatch.setenv("PT_BRICK", "3")
    w = phantom.tube()
    t = pt.Tracker(0)
    try:
        with pytest.raises(pt.PtError, match="PT_BRICK"):
            t.load_volume(w.volume)
    finally:
        t.close()


# ----------------------------------------------------------------------------- full size, sampled

@pytest.mark.parametrize("cfg", ["c3", "c4"])
def test_timed_instantiation_map_vs_oracle(pt, tracker, cfg):
    """The exact launch bench.py times (flags = 0: no per-particle outputs, compile-time
    16^3-brick layout, Morton claims) on configs[2] / [3]: every 16th WM seed at the full
    P = 5000, the FULL uint32 map compared with the oracle's bit for bit, and the kernel's
    step counter with the oracle's total."""
    import torch
    w = phantom.wm_seeds(phantom.config(cfg), every=16)
    tracker.load_volume(w.volume)
    m = tracker.track_workload(w, flags=0)
    torch.cuda.synchronize()
    st = tracker.stats()
    gm = m.cpu().numpy().view(np.uint32)
    r = oracle.track(w, want_particles=False, threads=_threads())
    assert np.array_equal(gm.astype(np.uint64), r["map"]), \
        f"{np.count_nonzero(gm.astype(np.uint64) != r['map'])} map cells differ"
    assert st["total_steps"] == int(r["map"].sum())
    assert st["particles"] == w.nparticles


@pytest.mark.parametrize("step", [0.5, 7.9, 14.5, 15.5, 40.0])
@pytest.mark.parametrize("half", [False, True])
def test_margin_bricks_and_bounds(pt, tracker, step, half):
    """The bench launch on the margin-padded brick layout: while step * max|v| <
    15 voxels the kernel takes no bounds test and leaving the volume is caught by the
    sentinel records of the margin / ragged bricks; above that the bounds-checked
    instantiation runs.  Large steps make particles leave the volume on every side, from
    ragged (non-multiple-of-16) edges: the map and the step counter must equal the oracle's."""
    import torch
    w = phantom.crossing(nx=45, ny=37, nz=21, lo=10, hi=30, zlo=3, zhi=18, sigma=0.4, f_jitter=0.05,
                         nseeds=96, particles_per_seed=64, nsamples=12)
    w = w.replace(step=step, max_steps=400)
    if half:
        w = phantom.to_half(w)
    tracker.load_volume(w.volume)
    m = tracker.track_workload(w, flags=0)
    torch.cuda.synchronize()
    st = tracker.stats()
    gm = m.cpu().numpy().view(np.uint32)
    r = oracle.track(w, want_particles=False)
    assert np.array_equal(gm.astype(np.uint64), r["map"]), \
        f"{np.count_nonzero(gm.astype(np.uint64) != r['map'])} map cells differ"
    assert st["total_steps"] == int(r["map"].sum())
    # and per particle through the outputs instantiation (bounds-checked, runtime layout)
    g = gpu_run(tracker, w)
    ro = oracle.track(w)
    assert_parity(g, ro)


@pytest.mark.parametrize("cfg", ["c2", "c2_dispersed"])
def test_timed_instantiation_full_config(pt, tracker, cfg):
    """configs[1] in the bench launch (flags = 0): the full map bit-exact vs the oracle."""
    import torch
    w = phantom.config(cfg)
    tracker.load_volume(w.volume)
    m = tracker.track_workload(w, flags=0)
    torch.cuda.synchronize()
    r = oracle.track(w, want_particles=False, threads=_threads())
    assert np.array_equal(m.cpu().numpy().view(np.uint32).astype(np.uint64), r["map"])
    assert tracker.stats()["total_steps"] == int(r["map"].sum())


@pytest.mark.parametrize("cfg", ["c3", "c4"])
def test_whole_brain_full_size_sampled(pt, tracker, cfg):
    """configs[2]/[3] at full size (all WM seeds x 5000 particles): the map of the bench
    launch (flags = 0) equals the map of the outputs instantiation bit for bit, and 3000
    sampled particles of the latter are recomputed one by one by the oracle, plus the global
    invariants at full size."""
    import torch
    w = phantom.config(cfg)
    tracker.load_volume(w.volume)
    m0 = tracker.track_workload(w, flags=0).clone()
    torch.cuda.synchronize()
    steps0 = tracker.stats()["total_steps"]
    m = tracker.track_workload(w, flags=REC_ALL)
    torch.cuda.synchronize()
    assert torch.equal(m0, m) and tracker.stats()["total_steps"] == steps0
    st = tracker.stats()
    out = tracker.get_paths(on_device=True)
    nst = out["nsteps"].to(torch.int64)
    total = int(nst.sum().item())
    gm = m.cpu().numpy().view(np.uint32)
    assert st["particles"] == w.nparticles
    assert st["total_steps"] == total == int(gm.sum(dtype=np.uint64))
    assert int(nst.max().item()) <= w.max_steps
    assert np.all(gm[w.volume.mask == 0] == 0)
    rng = np.random.default_rng(2012)
    pick = np.sort(rng.choice(w.nparticles, 3000, replace=False))
    P = w.particles_per_seed
    idx_t = torch.as_tensor(pick, device=out["nsteps"].device)
    g = {"nsteps": out["nsteps"][idx_t].cpu().numpy().view(np.uint16),
         "reason": out["reason"][idx_t].cpu().numpy(),
         "end": out["end"][idx_t].cpu().numpy()}
    rn, rr, re_ = [], [], []
    for li in pick:
        si, j = divmod(int(li), P)
        sub = w.replace(seeds=w.seeds[si:si + 1], seed_ids=w.ids()[si:si + 1])
        r = oracle.track(sub, j, j + 1, want_map=False)
        rn.append(r["nsteps"][0])
        rr.append(r["reason"][0])
        re_.append(r["end"][0])
    r = {"nsteps": np.array(rn), "reason": np.array(rr), "end": np.array(re_)}
    diverged = (g["nsteps"].astype(np.int64) != r["nsteps"]) | (g["reason"] != r["reason"]) | \
        np.any(g["end"].view(np.uint32) != r["end"].view(np.uint32), axis=1)
    assert diverged.sum() == 0, f"{diverged.sum()} of {len(pick)} sampled streamlines diverge"
    assert r["nsteps"].mean() > 10


# ----------------------------------------------------------------------------- NEXT-2 unique map

def _unique_run(pt, tr, w, extra=0):
    import torch
    tr.load_volume(w.volume)
    m = tr.track_workload(w, flags=pt.PT_MAP_UNIQUE | extra)
    torch.cuda.synchronize()
    return m.cpu().numpy().view(np.uint32), tr.stats()


@pytest.mark.parametrize("cfg", ["c2", "c2_dispersed"])
def test_unique_map_full_config(pt, tracker, cfg):
    """PT_MAP_UNIQUE (R25): configs[1] at full size, map bit-exact vs the oracle's
    per-streamline-unique map; the overflow check balances on the unique counts."""
    w = phantom.config(cfg)
    gm, st = _unique_run(pt, tracker, w)
    r = oracle.track(w, want_particles=False, want_unique=True, threads=_threads())
    assert np.array_equal(gm.astype(np.uint64), r["umap"])
    assert st["unique_visits"] == int(r["umap"].sum()) and st["total_steps"] == int(r["map"].sum())
    assert st["overflow"] == 0


@pytest.mark.parametrize("rec", [False, True])
@pytest.mark.parametrize("variant", [0, 1, 2])
def test_unique_map_loops_and_variants(pt, tracker, variant, rec):
    """Closed loops (vortex: streamlines revisit their voxels ~3 times), with and without the
    NEXT-3 variants (bidirectional union of halves, interpolation + f-weighted first fibre)
    and with per-particle outputs recorded on the side."""
    w = phantom.vortex(sigma=0.2, particles_per_seed=64, max_steps=700)
    w = w.replace(bidir=int(variant >= 1), interp=int(variant == 2), init_fibre=2 if variant == 2 else 0)
    flags = pt.PT_REC_LEN if rec else 0
    gm, st = _unique_run(pt, tracker, w, flags | pt.variant_flags(w.bidir, w.interp, w.init_fibre))
    r = oracle.track(w, want_unique=True, threads=_threads())
    assert np.array_equal(gm.astype(np.uint64), r["umap"])
    assert r["map"].sum() > 1.5 * r["umap"].sum()
    if rec:
        g = tracker.get_paths(nsteps=True, reason=False, end=False)
        assert np.array_equal(g["nsteps"].astype(np.int64), r["nsteps"].astype(np.int64))


def test_unique_map_whole_brain_sampled(pt, tracker):
    """configs[2] shape: every 64th WM seed at full P, unique map bit-exact vs the oracle;
    and a small hash-set budget (fewer persistent CTAs) gives the same map."""
    import os as _os
    w = phantom.wm_seeds(phantom.config("c3"), every=64)
    gm, st = _unique_run(pt, tracker, w)
    r = oracle.track(w, want_particles=False, want_unique=True, threads=_threads())
    assert np.array_equal(gm.astype(np.uint64), r["umap"])
    _os.environ["PT_UNIQUE_MB"] = "64"
    try:
        gm2, _ = _unique_run(pt, tracker, w)
    finally:
        del _os.environ["PT_UNIQUE_MB"]
    assert np.array_equal(gm2, gm)


def test_unique_map_errors(pt, tracker):
    w = phantom.tube(particles_per_seed=4)
    tracker.load_volume(w.volume)
    for bad in (pt.PT_KERNEL_SIMPLE, pt.PT_KERNEL_SEGMENTED):
        with pytest.raises(pt.PtError) as e:
            tracker.track_workload(w, flags=pt.PT_MAP_UNIQUE | bad)
        assert e.value.status == pt.PT_ERR_ARG


def test_c5_hcp_scale_sampled(pt, tracker):
    """configs[4] (HCP-scale 145x174x145, 50 samples x 3 fibres, fp16 records (32-B records,
    one sector per step), 10^4 particles per seed): every 64th WM seed at full P, the global
    invariants and 1500 sampled particles recomputed one by one by the oracle."""
    import psutil
    import torch
    if psutil.virtual_memory().total < 40e9:
        pytest.skip("c5 generation needs ~14 GB of host memory")
    w = phantom.wm_seeds(phantom.config("c5"), every=64)
    tracker.load_volume(w.volume)
    m = tracker.track_workload(w, flags=REC_ALL)
    torch.cuda.synchronize()
    st = tracker.stats()
    out = tracker.get_paths(on_device=True)
    nst = out["nsteps"].to(torch.int64)
    gm = m.cpu().numpy().view(np.uint32)
    assert st["particles"] == w.nparticles
    assert st["total_steps"] == int(nst.sum().item()) == int(gm.sum(dtype=np.uint64))
    assert np.all(gm[w.volume.mask == 0] == 0)
    pick = np.sort(np.random.default_rng(55).choice(w.nparticles, 1500, replace=False))
    idx_t = torch.as_tensor(pick, device=out["nsteps"].device)
    g = {"nsteps": out["nsteps"][idx_t].cpu().numpy().view(np.uint16),
         "reason": out["reason"][idx_t].cpu().numpy(), "end": out["end"][idx_t].cpu().numpy()}
    P = w.particles_per_seed
    rn, rr, re_ = [], [], []
    for li in pick:
        si, j = divmod(int(li), P)
        r = oracle.track(w.replace(seeds=w.seeds[si:si + 1], seed_ids=w.ids()[si:si + 1]), j, j + 1,
                         want_map=False)
        rn.append(r["nsteps"][0])
        rr.append(r["reason"][0])
        re_.append(r["end"][0])
    assert np.array_equal(g["nsteps"].astype(np.int64), np.array(rn))
    assert np.array_equal(g["reason"], np.array(rr))
    assert np.array_equal(g["end"].view(np.uint32), np.array(re_).view(np.uint32))


# ----------------------------------------------------------------------------- invariances

def test_sharding_invariance(pt, tracker):
    """C-pin-10 on the GPU: seeds sharded i mod G (G = 2, 3) with global seed ids give the
    same per-pid results, and the shard maps sum to the unsharded map (what the NCCL
    reduce of the multi-GPU path computes)."""
    import torch
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=300, particles_per_seed=500)
    full = gpu_run(tracker, w)
    for G in (2, 3):
        tot = np.zeros_like(full["map"], dtype=np.uint64)
        for rank in range(G):
            sel = np.arange(rank, w.nseeds, G)
            sub = w.replace(seeds=w.seeds[sel].copy(), seed_ids=w.ids()[sel].copy())
            g = gpu_run(tracker, sub)
            tot += g["map"]
            rows = (sel[:, None] * w.particles_per_seed + np.arange(w.particles_per_seed)).ravel()
            assert np.array_equal(g["nsteps"], full["nsteps"][rows])
            assert np.array_equal(g["end"].view(np.uint32), full["end"][rows].view(np.uint32))
        assert np.array_equal(tot, full["map"].astype(np.uint64))
    torch.cuda.synchronize()


def test_host_buffers_and_accumulate(pt, tracker):
    """e2e path: host seeds + host map (H2D/D2H inside pt_track) equals the device path;
    PT_MAP_ACCUMULATE adds to the existing map."""
    w = phantom.crossing(sigma=0.15, nseeds=50, particles_per_seed=200)
    dev = gpu_run(tracker, w, 0)
    hm = np.zeros((w.volume.nz, w.volume.ny, w.volume.nx), np.uint32)
    tracker.track(w.seeds, None, step=w.step, curv_thr=w.curv_thr, fib_thr=w.fib_thr,
                  max_steps=w.max_steps, rng_seed=w.rng_seed, particles_per_seed=w.particles_per_seed,
                  out_map=hm)
    assert np.array_equal(hm, dev["map"])
    tracker.track(w.seeds, None, step=w.step, curv_thr=w.curv_thr, fib_thr=w.fib_thr,
                  max_steps=w.max_steps, rng_seed=w.rng_seed, particles_per_seed=w.particles_per_seed,
                  out_map=hm, flags=pt.PT_MAP_ACCUMULATE)
    assert np.array_equal(hm, 2 * dev["map"])


def test_overflow_is_detected(pt, tracker):
    """R17: a uint32 cell wrapping past 2^32-1 is reported as PT_ERR_OVERFLOW."""
    import torch
    w = phantom.tube(particles_per_seed=10)
    tracker.load_volume(w.volume)
    m = torch.full((w.volume.nz, w.volume.ny, w.volume.nx), -3, dtype=torch.int32, device="cuda")
    tracker.track_workload(w, flags=pt.PT_MAP_ACCUMULATE, out_map=m)
    with pytest.raises(pt.PtError) as e:
        tracker.stats()
    assert e.value.status == pt.PT_ERR_OVERFLOW


# ----------------------------------------------------------------------------- edge cases

def test_edge_cases(pt, tracker):
    import torch
    w = phantom.crossing(sigma=0.15, nseeds=20, particles_per_seed=33)
    # seeds outside the volume and outside the mask (R12), plus max_steps = 1 and P = 1
    seeds = np.concatenate([w.seeds, np.array([[-5.0, 3.0, 3.0], [0.5, 0.5, 0.5], [70.0, 1.0, 1.0]],
                                              np.float32)])
    for kw in ({}, {"max_steps": 1}, {"particles_per_seed": 1}, {"max_steps": 3}):
        ww = w.replace(seeds=seeds, **kw)
        g = gpu_run(tracker, ww)
        r = oracle.track(ww)
        assert_parity(g, r)
    # no seeds: the map is zeroed, nothing else happens
    tracker.load_volume(w.volume)
    m = torch.full((w.volume.nz, w.volume.ny, w.volume.nx), 7, dtype=torch.int32, device="cuda")
    tracker.track_workload(w, seeds=np.zeros((0, 3), np.float32), out_map=m)
    torch.cuda.synchronize()
    assert int(m.abs().sum().item()) == 0
    assert tracker.stats()["particles"] == 0


def test_errors(pt):
    t = pt.Tracker(0)
    w = phantom.tube(particles_per_seed=4)
    with pytest.raises(pt.PtError) as e:
        t.track_workload(w)
    assert e.value.status == pt.PT_ERR_STATE
    t.load_volume(w.volume)
    for bad in ({"max_steps": 0}, {"max_steps": 70000}, {"step": 0.0}, {"curv_thr": 1.5},
                {"particles_per_seed": 0}):
        with pytest.raises(pt.PtError) as e:
            t.track_workload(w.replace(**bad))
        assert e.value.status == pt.PT_ERR_ARG
    v = w.volume
    dy = v.dyads.copy()
    dy[0, 0, 8, 16, 16, 0] = np.nan  # inside the tube mask
    with pytest.raises(pt.PtError) as e:
        t.load_samples(dy, v.f, v.mask, v.nsamples, v.nfibres)
    assert e.value.status == pt.PT_ERR_ARG
    with pytest.raises(pt.PtError) as e:
        t.get_paths(paths=True)
    t.close()


def test_argument_checks(pt, tracker):
    """wrong dtypes are refused by the binding before a pointer crosses the ABI;
    labels above ntargets are PT_ERR_ARG (no out-of-bounds connectivity write); a
    device-resident seed id whose pids overflow 64 bits is reported as PT_ERR_ARG."""
    import torch
    w = phantom.crossing(sigma=0.15, nseeds=8, particles_per_seed=8)
    tracker.load_volume(w.volume)
    kw = dict(step=w.step, curv_thr=w.curv_thr, fib_thr=w.fib_thr, max_steps=w.max_steps,
              rng_seed=w.rng_seed, particles_per_seed=w.particles_per_seed)
    with pytest.raises(TypeError):
        tracker.track(w.seeds.astype(np.float64), None, **kw)
    with pytest.raises(TypeError):
        tracker.track(w.seeds, np.arange(w.nseeds, dtype=np.int32), **kw)
    with pytest.raises(ValueError):
        tracker.track(w.seeds[:, :2].copy(), None, **kw)
    v = w.volume
    with pytest.raises(TypeError):
        tracker.load_samples(v.dyads, v.f.astype(np.float16), v.mask, v.nsamples, v.nfibres)
    lab = np.zeros(v.mask.shape, np.uint8)
    lab[0, 0, 0] = 9
    with pytest.raises(pt.PtError) as e:
        tracker.load_targets(lab, 8)
    assert e.value.status == pt.PT_ERR_ARG
    tracker.load_targets(lab, 9)
    big = torch.full((w.nseeds,), -1, dtype=torch.int64, device="cuda")  # 2^64 - 1
    tracker.track(torch.as_tensor(w.seeds, device="cuda"), big, **kw)
    with pytest.raises(pt.PtError) as e:
        tracker.stats()
    assert e.value.status == pt.PT_ERR_ARG


def test_lane_efficiency_and_gather_bench(pt, tracker):
    """Lane refill keeps warps converged: active-lane fraction of the persistent kernel is
    well above the no-refill ablation's (~1/H_32 for exponential lengths)."""
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=400, particles_per_seed=2000)
    a = gpu_run(tracker, w, 0)["stats"]
    b = gpu_run(tracker, w, pt.PT_KERNEL_SIMPLE)["stats"]
    fa = a["lane_active"] / a["lane_slots"]
    fb = b["lane_active"] / b["lane_slots"]
    assert a["total_steps"] == b["total_steps"]
    assert fa > 0.8 and fa > fb, (fa, fb)
    r = tracker.gather_bench(1 << 30, 32)
    assert r > 1e9


# ----------------------------------------------------------------------------- NEXT-1 paper mode

def test_paper_mode_closed_form(pt, tracker):
    """NEXT-1 on the GPU: the alternating-sample tube of the oracle pin, bit-exact."""
    from tests.test_oracle_pins import _alternating_tube
    w = _alternating_tube(P=64)
    g = gpu_run(tracker, w)
    r = oracle.track(w)
    assert_parity(g, r)


@pytest.mark.parametrize("half", [False, True])
def test_paper_mode_parity(pt, tracker, half):
    """NEXT-1: one sample volume per streamline (P = S), every particle and the map, plus
    paths, on a small paper-dataset-shaped volume."""
    w = phantom.paper_dataset(1, 0.2, 0.8)
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 1500))
    if half:
        w = phantom.to_half(w)
    g = gpu_run(tracker, w, REC_ALL | pt.PT_REC_PATHS, path_stride=256)
    r = oracle.track(w, path_stride=256, threads=_threads())
    assert_parity(g, r)
    assert paths_equal(g["paths"], r["paths"])
    s = gpu_run(tracker, w, REC_ALL | pt.PT_KERNEL_SIMPLE)
    assert_parity(s, r)


# ----------------------------------------------------------------------------- NEXT-2 connectivity

def _targets(shape, n, seed):
    """n roughly spherical target regions at random positions (labels 1..n)."""
    rng = np.random.default_rng(seed)
    Z, Y, X = shape
    zz, yy, xx = np.meshgrid(np.arange(Z), np.arange(Y), np.arange(X), indexing="ij")
    lab = np.zeros(shape, np.uint8)
    for t in range(n):
        c = rng.uniform([0, 0, 0], [Z, Y, X])
        r = rng.uniform(2.0, 6.0)
        lab[(zz - c[0]) ** 2 + (yy - c[1]) ** 2 + (xx - c[2]) ** 2 < r * r] = t + 1
    return lab


@pytest.mark.parametrize("simple", [False, True])
@pytest.mark.parametrize("mode", [0, 1])
def test_connectivity_parity(pt, tracker, simple, mode):
    """NEXT-2: seed x target matrix bit-exact vs the oracle, both kernels, random
    per-step sampling and paper mode."""
    import torch
    w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=200, particles_per_seed=300).replace(sample_mode=mode)
    lab = _targets(w.volume.mask.shape, 64, seed=7)
    tracker.load_volume(w.volume)
    tracker.load_targets(lab, 64)
    flags = REC_ALL | pt.PT_REC_CONN | (pt.PT_KERNEL_SIMPLE if simple else 0)
    m = tracker.track_workload(w, flags=flags)
    torch.cuda.synchronize()
    g = tracker.get_paths()
    g["map"] = m.cpu().numpy().view(np.uint32)
    conn = tracker.connectivity().reshape(w.nseeds, 64)
    r = oracle.track(w, labels=lab, ntargets=64, threads=_threads())
    assert_parity(g, r)
    assert np.array_equal(conn.astype(np.uint64), r["conn"])
    assert conn.sum() > 1000


def test_connectivity_brain_and_errors(pt, tracker):
    w = phantom.whole_brain(nx=40, ny=36, nz=24, semi=(17.0, 15.0, 10.0), nsamples=16, nfibres=3,
                            particles_per_seed=37)
    w = phantom.wm_seeds(w, every=max(1, w.nseeds // 200))
    lab = _targets(w.volume.mask.shape, 12, seed=3)
    tracker.load_volume(w.volume)
    with pytest.raises(pt.PtError) as e:
        tracker.track_workload(w, flags=pt.PT_REC_CONN)
    assert e.value.status == pt.PT_ERR_STATE
    with pytest.raises(pt.PtError) as e:
        tracker.load_targets(lab, 65)
    assert e.value.status == pt.PT_ERR_ARG
    tracker.load_targets(lab, 12)
    tracker.track_workload(w, flags=pt.PT_REC_CONN)
    conn = tracker.connectivity().reshape(w.nseeds, 12)
    r = oracle.track(w, labels=lab, ntargets=12, want_particles=False)
    assert np.array_equal(conn.astype(np.uint64), r["conn"])
