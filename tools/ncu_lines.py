"""Per-source-line warp-stall attribution from an ncu report (needs -lineinfo).

usage: python tools/ncu_lines.py report.ncu-rep [top]
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source",
                          "cuda,sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    agg = defaultdict(float)
    src = {}
    fname = "?"
    cur_line = None
    for r in rows:
        if len(r) >= 2 and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if len(r) < 6 or r[0] in ("Line No", "Function Name"):
            continue
        if r[0] not in ("", "-") and r[2] in ("-",):
            cur_line = (fname, r[0])
            src[cur_line] = r[1]
            try:
                agg[cur_line] += float(r[4])
            except ValueError:
                pass
    tot = sum(agg.values()) or 1.0
    for (f, ln), w in sorted(agg.items(), key=lambda x: -x[1])[:top]:
        print(f"{100 * w / tot:5.1f}%  {f}:{ln}  {src[(f, ln)][:100]}")


if __name__ == "__main__":
    main()
