"""Warp-stall samples of a kernel aggregated per CUDA source line (ncu source page, cuda,sass).

    python tools/ncu_lines.py report.ncu-rep k_step [top]
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict


def main(path, kernel, top=30):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "-k", f"regex:{kernel}"], capture_output=True, text=True).stdout
    agg = defaultdict(lambda: [0, 0, ""])
    fname, hdr, cur = "?", None, None
    for row in csv.reader(io.StringIO(out)):
        if not row:
            continue
        if row[0] == "File Path":
            fname = row[1].rsplit("/", 1)[-1]
            continue
        if row[0] == "Line No":
            hdr = row
            si = hdr.index("Warp Stall Sampling (All Samples)")
            ie = hdr.index("Instructions Executed")
            continue
        if hdr is None or row[0] == "Function Name":
            continue
        if row[0]:   # a CUDA source line
            cur = (fname, int(row[0]))
            agg[cur][2] = row[1].strip()
        elif cur is not None:
            try:
                agg[cur][0] += int(row[si] or 0)
                agg[cur][1] += int(row[ie] or 0)
            except ValueError:
                pass
    tot = sum(v[0] for v in agg.values()) or 1
    for (f, ln), (s, e, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[: int(top)]:
        print(f"{100.0 * s / tot:5.1f}%  {e:>10d}  {f}:{ln:<5d} {src[:90]}")


if __name__ == "__main__":
    main(*sys.argv[1:])
