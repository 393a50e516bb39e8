"""SURVEY §8(d) ablations on one workload, generated once (one process, one GPU):

  (i)   no lane refill, one thread per particle (PT_KERNEL_SIMPLE; the paper's A_MaxStep /
        "Extreme case 1")
  (ii)  segmented relaunch with device compaction (PT_KERNEL_SEGMENTED), the paper's
        schedules A_1, A_10, A_50, strategy B and C (Table IV)
  (iii) fp32 vs fp16 records (c3 vs c4)
  (v)   raster vs Morton seed order (PT_SEED_ORDER_INPUT)
  (vi)  raster vs bricked record layout (PT_BRICK=0 vs the default 16^3 bricks)
  plus the NEXT-3 variant instantiation on the default semantics (PT_KERNEL_VARIANT), the
  variants themselves (PT_BIDIR, PT_INTERP) and the NEXT-2 unique map (PT_MAP_UNIQUE).

Every run's total steps must equal the main kernel's (same parity contract: the results
are identical, only the schedule differs).  Prints one JSON line per variant and a markdown
table on stdout.

  python scripts/ablations.py [--config c3] [--reps 2] [--seed-every 1]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c3")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--seed-every", type=int, default=1)
    ap.add_argument("--only", default="", help="comma list of substrings of the variant names to run")
    args = ap.parse_args()
    import numpy as np
    import torch

    import paper_conf_ipps_xuzwrwxgxy12_b200 as pt
    import phantom

    w = phantom.config(args.config)
    if args.seed_every > 1:
        w = phantom.wm_seeds(w, every=args.seed_every)
    tr = pt.Tracker(0)
    dev = torch.device("cuda", 0)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)
    seeds = torch.as_tensor(w.seeds, device=dev).contiguous()
    ids = torch.as_tensor(w.ids().astype(np.int64), device=dev).contiguous()
    out_map = torch.empty((w.volume.nz, w.volume.ny, w.volume.nx), dtype=torch.int32, device=dev)

    variants = [
        ("main (persistent, lane refill, Morton)", 0, None, w),
        ("(v) raster seed order", pt.PT_SEED_ORDER_INPUT, None, w),
        ("variant instantiation, default semantics", pt.PT_KERNEL_VARIANT, None, w),
        ("NEXT-3 bidirectional", pt.PT_BIDIR, None, w),
        ("NEXT-3 probabilistic interpolation", pt.PT_INTERP, None, w),
        ("NEXT-3 bidirectional + interpolation + f-weighted first fibre",
         pt.PT_BIDIR | pt.PT_INTERP | pt.PT_INIT_FWEIGHT, None, w),
        ("NEXT-2 per-streamline-unique map", pt.PT_MAP_UNIQUE, None, w),
        ("(i) no refill, one thread per particle (A_MaxStep)", pt.PT_KERNEL_SIMPLE, None, w),
        ("(ii) segmented A_1", pt.PT_KERNEL_SEGMENTED, (1,), w),
        ("(ii) segmented A_10", pt.PT_KERNEL_SEGMENTED, (10,), w),
        ("(ii) segmented A_50", pt.PT_KERNEL_SEGMENTED, (50,), w),
        ("(ii) segmented strategy B", pt.PT_KERNEL_SEGMENTED, pt.SEGMENTS_B, w),
        ("(ii) segmented strategy C", pt.PT_KERNEL_SEGMENTED, pt.SEGMENTS_C, w),
        ("(ii) segmented A_2000 (one segment)", pt.PT_KERNEL_SEGMENTED, (2000,), w),
    ]
    variants = [v + ("4",) for v in variants]
    variants.insert(1, ("(vi) raster record layout (PT_BRICK=0)", 0, None, w, "0"))
    variants.append(("(vi) raster record layout, no refill (PT_BRICK=0)", pt.PT_KERNEL_SIMPLE, None, w, "0"))
    if args.config == "c3" and not args.only:
        variants.append(("(iii) fp16 records (c4)", 0, None, None, "4"))
    rows = []
    ref_steps = None
    loaded = None
    for name, flags, sched, wv, brick in variants:
        if args.only and not any(o and o in name for o in args.only.split(",")):
            continue
        if wv is None:
            wv = phantom.to_half(w)
        if loaded != (id(wv), brick):
            os.environ["PT_BRICK"] = brick  # read by pt_load_samples
            tr.load_volume(wv.volume)
            loaded = (id(wv), brick)
        if sched:
            tr.set_segments(sched)
        best = None
        for rep in range(args.reps + 1):
            flush.fill_(1)
            tr.track(seeds, ids, step=wv.step, curv_thr=wv.curv_thr, fib_thr=wv.fib_thr,
                     max_steps=wv.max_steps, rng_seed=wv.rng_seed,
                     particles_per_seed=wv.particles_per_seed, out_map=out_map, flags=flags)
            torch.cuda.synchronize()
            st = tr.stats()
            if rep > 0 and (best is None or st["track_ms"] < best["track_ms"]):
                best = st
        if ref_steps is None:
            ref_steps = best["total_steps"]
        ok = best["total_steps"] == ref_steps
        r = {"variant": name, "flags": flags, "schedule": list(sched) if sched else None,
             "track_ms": best["track_ms"], "kernel_ms": best["kernel_ms"],
             "steps_per_s": best["total_steps"] / (best["track_ms"] * 1e-3),
             "active_lane_fraction": best["lane_active"] / max(1, best["lane_slots"]),
             "total_steps": best["total_steps"], "same_steps_as_main": ok}
        rows.append(r)
        print(json.dumps(r), flush=True)
    print(f"\n| variant | pass ms | steps/s | vs main | active-lane fraction | same total steps |")
    print("|---|---|---|---|---|---|")
    base = rows[0]["steps_per_s"]
    for r in rows:
        print(f"| {r['variant']} | {r['track_ms']:.0f} | {r['steps_per_s'] / 1e9:.1f} G | "
              f"{r['steps_per_s'] / base:.2f}x | {r['active_lane_fraction']:.3f} | {r['same_steps_as_main']} |")
    tr.close()


if __name__ == "__main__":
    main()
