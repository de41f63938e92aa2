"""Summarise an ncu launch list (gpu__time_duration.sum per launch) per kernel.
usage: python tools/launches.py gpurun_out/launches_<tag>.csv [last_n]"""
import collections
import csv
import re
import sys


def main(path, last=None):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h, rows = rows[hi], rows[hi + 1:]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    seq = []
    for r in rows:
        name = re.sub(r"\(.*", "", r[ki]).replace("void ", "")
        name = re.sub(r"glb::|\(anonymous namespace\)::|unnamed>::", "", name)
        seq.append((name, float(r[vi].replace(",", "")) / 1e3))
    if last:
        seq = seq[-int(last):]
    agg = collections.OrderedDict()
    for n, t in seq:
        a = agg.setdefault(n, [0, 0.0])
        a[0] += 1
        a[1] += t
    tot = sum(a[1] for a in agg.values())
    print(f"{'kernel':40s} {'launches':>8s} {'mean us':>9s} {'total us':>10s} {'share':>6s}")
    for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{n:40s} {c:8d} {t / c:9.2f} {t:10.1f} {100 * t / tot:5.1f}%")


if __name__ == "__main__":
    main(*sys.argv[1:])
