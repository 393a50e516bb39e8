"""Summarise an ncu capture of the MCMC kernel into profiles/<tag>_mcmc_ncu.md.

  python scripts/ncu_mcmc_summary.py --rep gpurun_out/prof_mcmc_m2prof.ncu-rep --tag r01f \
      --voxels 50277 --loops 600 --note "..."

Reports the executed FP64 lane-instructions per voxel-loop (DFMA + DMUL + DADD), which
bench.py uses as the per-unit figure of the MCMC roofline (bound "alu", FP64 pipe).
"""
from __future__ import annotations

import argparse
import csv
import io
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = [
    ("gpu__time_duration.sum", "kernel duration"),
    ("launch__registers_per_thread", "registers per thread"),
    ("sm__warps_active.avg.per_cycle_active", "active warps per SM"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "FP64 pipe active % of peak"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe % of peak"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe % of peak"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "XU (SFU) pipe % of peak"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe % of peak"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads per warp instruction (/32)"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("smsp__sass_thread_inst_executed_op_dfma_pred_on.sum", "DFMA lane-instructions"),
    ("smsp__sass_thread_inst_executed_op_dmul_pred_on.sum", "DMUL lane-instructions"),
    ("smsp__sass_thread_inst_executed_op_dadd_pred_on.sum", "DADD lane-instructions"),
    ("smsp__average_warp_latency_per_inst_issued.ratio", "cycles per issued instruction per warp"),
    ("smsp__average_warps_issue_stalled_wait_per_issue_active.ratio", "stall: wait (fixed latency)"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall: short scoreboard"),
    ("smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio", "stall: not selected"),
    ("smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio", "stall: math pipe throttle"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall: long scoreboard"),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rep", required=True)
    ap.add_argument("--tag", required=True)
    ap.add_argument("--voxels", type=int, required=True)
    ap.add_argument("--loops", type=int, required=True)
    ap.add_argument("--note", default="")
    args = ap.parse_args()
    out = subprocess.run(["ncu", "-i", args.rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    get = {h: (v, u) for h, u, v in zip(hdr, units, vals)}
    lines = [f"# {args.tag}: ncu capture of the MCMC kernel", "", args.note, "",
             f"`{os.path.relpath(args.rep, ROOT)}`; {args.voxels} voxels x {args.loops} loops.", "",
             "| counter | value |", "|---|---|"]
    for k, name in KEYS:
        if k in get:
            v, u = get[k]
            lines.append(f"| {name} (`{k}`) | {v} {u} |")
    try:
        dp = sum(float(get[k][0].replace(",", "")) for k in (
            "smsp__sass_thread_inst_executed_op_dfma_pred_on.sum",
            "smsp__sass_thread_inst_executed_op_dmul_pred_on.sum",
            "smsp__sass_thread_inst_executed_op_dadd_pred_on.sum"))
        per = dp / (args.voxels * args.loops)
        lines += ["", f"FP64 lane-instructions (DFMA + DMUL + DADD) per voxel-loop: **{per:.0f}**"]
    except (KeyError, ValueError):
        pass
    path = os.path.join(ROOT, "profiles", f"{args.tag}_mcmc_ncu.md")
    open(path, "w").write("\n".join(lines) + "\n")
    print(open(path).read())


if __name__ == "__main__":
    main()
