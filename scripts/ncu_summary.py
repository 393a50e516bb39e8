"""Summarise ncu outputs brought back in gpurun_out/ into profiles/ (tracked).

  python scripts/ncu_summary.py --tag r01 --cfg c3 [--launches gpurun_out/launches_c3_r01.csv]
         [--rep gpurun_out/prof_c3_r01.ncu-rep]

Writes profiles/<tag>_<cfg>_launches.md (per-kernel share of the launch list) and
profiles/<tag>_<cfg>_track_ncu.md (key counters of the --set full capture), and updates
profiles/ncu_track_summary.json (dram bytes per launch -> bench.py roofline.traffic).
"""
from __future__ import annotations

import argparse
import collections
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")

KEYS = [
    ("gpu__time_duration.sum", "kernel duration"),
    ("dram__bytes_read.sum", "DRAM bytes read"),
    ("dram__bytes_write.sum", "DRAM bytes written"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 sector hit rate"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2 read sectors (from L1/tex)"),
    ("lts__t_sectors_srcunit_tex_op_red.sum", "L2 reduction sectors (map RED)"),
    ("lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum", "L2 read sectors that hit"),
    ("lts__t_sectors_srcunit_tex_op_red_lookup_miss.sum", "L2 RED sectors that missed"),
    ("lts__t_requests_srcunit_tex_op_read.sum", "L2 read requests (from L1/tex)"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "L1 global load sectors requested"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld_lookup_hit.sum", "L1 global load sectors that hit"),
    ("l1tex__m_xbar2l1tex_read_sectors_mem_lg_op_ld.sum", "sectors L2 -> L1 (global loads)"),
    ("dram__sectors_read.sum", "DRAM sectors read"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput % of peak"),
    ("l1tex__t_sector_hit_rate.pct", "L1 sector hit rate"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "L1 throughput % of peak"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads per warp instruction (/32)"),
    ("sm__warps_active.avg.per_cycle_active", "active warps per SM"),
    ("launch__registers_per_thread", "registers per thread"),
    ("launch__grid_size", "grid size"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock"),
    ("smsp__average_warp_latency_per_inst_issued.ratio", "cycles per issued instruction per warp"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall: long scoreboard"),
    ("smsp__average_warps_issue_stalled_wait_per_issue_active.ratio", "stall: wait"),
    ("smsp__average_warps_issue_stalled_branch_resolving_per_issue_active.ratio", "stall: branch resolving"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall: short scoreboard"),
    ("smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio", "stall: lg throttle"),
]


def launches(path):
    rows = [r for r in csv.reader(open(path)) if r and not r[0].startswith("==")]
    hdr = rows[0]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "s": 1e3, "second": 1e3}
    tot, cnt = collections.defaultdict(float), collections.Counter()
    for r in rows[1:]:
        try:
            v = float(r[vi].replace(",", "")) * scale[r[ui]]
        except (ValueError, KeyError, IndexError):
            continue
        tot[r[ki]] += v
        cnt[r[ki]] += 1
    T = sum(tot.values())
    out = ["| kernel | launches | total ms | avg ms | share |", "|---|---|---|---|---|"]
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        out.append(f"| `{k[:90]}` | {cnt[k]} | {v:.3f} | {v / cnt[k]:.3f} | {100 * v / T:.2f}% |")
    return "\n".join(out), tot, cnt


def raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    return [{h: (v, u) for h, u, v in zip(hdr, units, r)} for r in rows[2:]]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", required=True)
    ap.add_argument("--cfg", required=True)
    ap.add_argument("--launches")
    ap.add_argument("--rep")
    ap.add_argument("--note", default="")
    ap.add_argument("--bench-log", help="stdout of the captured bench.py run (its JSON line gives the steps per launch)")
    ap.add_argument("--steps", type=float, help="committed steps of the captured launch (else from --bench-log)")
    a = ap.parse_args()
    os.makedirs(PROF, exist_ok=True)
    if a.launches:
        table, _, _ = launches(a.launches)
        with open(os.path.join(PROF, f"{a.tag}_{a.cfg}_launches.md"), "w") as f:
            f.write(f"# Launch list, {a.cfg} ({a.tag})\n\n`ncu --metrics gpu__time_duration.sum "
                    f"--clock-control none` of `bench.py --config {a.cfg} --steps 2 --warmup 1` "
                    f"(cold-cache, serialised: compare shares, not absolutes).\n\n{table}\n")
    if a.rep:
        recs = raw(a.rep)
        lines = [f"# ncu --set full: tracking kernel, {a.cfg} ({a.tag})", "", a.note, "",
                 "| counter | value | unit | meaning |", "|---|---|---|---|"]
        r = recs[0]
        for k, meaning in KEYS:
            if k in r:
                v, u = r[k]
                lines.append(f"| `{k}` | {v} | {u} | {meaning} |")
        with open(os.path.join(PROF, f"{a.tag}_{a.cfg}_track_ncu.md"), "w") as f:
            f.write("\n".join(lines) + "\n")
        sp = os.path.join(PROF, "ncu_track_summary.json")
        d = json.load(open(sp)) if os.path.exists(sp) else {"per_config": {}}

        def num(k):
            v, u = r[k]
            v = float(v.replace(",", ""))
            mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)
            return v * mult
        steps = a.steps
        if steps is None and a.bench_log:
            for ln in open(a.bench_log, errors="replace"):
                if ln.startswith("{") and '"steps_per_pass"' in ln:
                    cfgd = json.loads(ln)["config"]
                    steps = float(cfgd["steps_per_pass"])
        dram = num("dram__bytes_read.sum") + num("dram__bytes_write.sum")
        e = {
            "tag": a.tag,
            "dram_bytes_per_launch": dram,
            "l2_hit_rate_pct": float(r["lts__t_sector_hit_rate.pct"][0]),
            "l1_hit_rate_pct": float(r["l1tex__t_sector_hit_rate.pct"][0]),
            "kernel_s_under_ncu": float(r["gpu__time_duration.sum"][0]),
            "issue_active_pct": float(r["smsp__issue_active.avg.pct_of_peak_sustained_active"][0]),
            # warp execution efficiency: active threads per executed warp instruction / 32
            "warp_exec_efficiency": float(r["smsp__thread_inst_executed_per_inst_executed.ratio"][0]) / 32.0,
            "lts_throughput_pct": float(r["lts__throughput.avg.pct_of_peak_sustained_elapsed"][0]),
        }
        if steps:
            e["steps_per_launch_captured"] = steps
            e["dram_bytes_per_step"] = dram / steps
            # warp instructions per 32 committed steps (= per fully active warp-step)
            e["warp_inst_per_32_steps"] = 32.0 * num("smsp__inst_executed.sum") / steps
            e["l2_read_sectors_per_step"] = num("lts__t_sectors_srcunit_tex_op_read.sum") / steps
            e["l2_red_sectors_per_step"] = num("lts__t_sectors_srcunit_tex_op_red.sum") / steps
        if a.note:
            e["note"] = a.note
        d["per_config"][a.cfg] = e
        json.dump(d, open(sp, "w"), indent=1)
    print("ok")


if __name__ == "__main__":
    main()
