"""Summarise an ncu `--metrics gpu__time_duration.sum --csv` launch list: per kernel
name, launch count, mean duration and share of the summed kernel time.
Usage: python scripts/launch_summary.py launches.csv "<command line it came from>" [note]"""
import collections
import csv
import sys


def summarise(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.reader(lines))
    hdr = rows[0]
    ik, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    scale = {"ns": 1.0, "nsecond": 1.0, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}
    acc = collections.OrderedDict()
    for r in rows[1:]:
        if r[ik] == "Kernel Name":
            continue
        ns = float(r[iv].replace(",", "")) * scale.get(r[iu], 1.0)
        acc.setdefault(r[ik], []).append(ns)
    total = sum(sum(v) for v in acc.values())
    return [(k, len(v), sum(v) / len(v), sum(v) / total) for k, v in sorted(acc.items(), key=lambda kv: -sum(kv[1]))]


if __name__ == "__main__":
    print(sys.argv[2] if len(sys.argv) > 2 else "")
    if len(sys.argv) > 3:
        print(sys.argv[3])
    for k, n, mean, share in summarise(sys.argv[1]):
        print(f"{k[:90]}: launches={n} mean_ns={mean:.0f} share={share:.3f}")
