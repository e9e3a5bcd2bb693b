"""Summarise an `ncu --csv --log-file` launch list: per kernel count, mean duration, share."""
import csv
import sys
from collections import defaultdict


def main(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.reader(lines[start:]))
    hdr = rows[0]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    d = defaultdict(list)
    for r in rows[1:]:
        if len(r) > vi and r[mi] == "gpu__time_duration.sum":
            d[r[ki].split("(")[0]].append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in d.values())
    print(f"{'kernel':50s} {'launches':>8s} {'mean':>10s} {'share':>7s}")
    for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1])):
        print(f"{k[:50]:50s} {len(v):8d} {sum(v) / len(v):10.2f} {100 * sum(v) / tot:6.1f}%")


if __name__ == "__main__":
    main(sys.argv[1])
