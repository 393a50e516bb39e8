"""Where the warps of a captured kernel wait, per SASS instruction (ncu --page source).

  python scripts/ncu_source_summary.py REP.ncu-rep OUT.md [--title T]

Writes the total warp-stall samples, the share of the top instructions and the share
of the instructions that first consume a record gather (ISETP on the sentinel word)."""
from __future__ import annotations

import csv
import io
import subprocess
import sys


def main():
    rep, out = sys.argv[1], sys.argv[2]
    title = sys.argv[4] if len(sys.argv) > 4 and sys.argv[3] == "--title" else rep
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr = rows[1]
    data = rows[2:]
    iS, iE = hdr.index("Source"), hdr.index("Instructions Executed")
    iW = hdr.index("Warp Stall Sampling (All Samples)")
    recs = [(r[iS].strip(), int(r[iE] or 0), int(r[iW] or 0)) for r in data]
    tot_w = sum(w for _, _, w in recs)
    tot_e = sum(e for _, e, _ in recs)
    gather_use = sum(w for s, _, w in recs if s.startswith("ISETP") and "-0x1" in s)
    lines = [f"# Warp-stall samples per SASS instruction: {title}", "",
             f"{len(recs)} SASS instructions, {tot_e:,} warp instructions executed, {tot_w:,} stall samples.", "",
             f"First consumers of a record gather (`ISETP ... -0x1`, the sentinel test of word 3): "
             f"**{100.0 * gather_use / max(tot_w, 1):.1f} %** of all samples.", "",
             "| rank | instruction | executed | samples | share |", "|---|---|---|---|---|"]
    for k, (s, e, w) in enumerate(sorted(recs, key=lambda t: -t[2])[:20]):
        lines.append(f"| {k + 1} | `{s}` | {e:,} | {w:,} | {100.0 * w / max(tot_w, 1):.2f} % |")
    open(out, "w").write("\n".join(lines) + "\n")
    print("ok", out)


if __name__ == "__main__":
    main()
