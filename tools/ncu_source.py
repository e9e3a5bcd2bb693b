"""Top stall lines of a kernel from an ncu report's source page (SASS view)."""
import csv
import io
import subprocess
import sys


def main(path, kernel, top=25):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "-k", f"regex:{kernel}"],
                         capture_output=True, text=True).stdout
    lines = out.splitlines()
    # first line: kernel name; second: header
    rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
    hdr = rows[0]
    si = hdr.index("Warp Stall Sampling (All Samples)")
    src = hdr.index("Source")
    ex = hdr.index("Instructions Executed")
    data = []
    for r in rows[1:]:
        try:
            data.append((int(r[si]), r[src].strip(), r[ex]))
        except Exception:
            pass
    tot = sum(d[0] for d in data) or 1
    for s, code, e in sorted(data, reverse=True)[: int(top)]:
        print(f"{100.0 * s / tot:5.1f}%  {e:>10s}  {code[:110]}")


if __name__ == "__main__":
    main(*sys.argv[1:])
