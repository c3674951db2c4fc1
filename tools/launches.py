"""Summarise an ncu launch-list CSV (--metrics gpu__time_duration.sum): per-launch sequence
(-v) and per-kernel totals."""
import collections
import csv
import sys


def main(path, verbose=False):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    h = rows[0]
    ki, vi, gi = h.index('Kernel Name'), h.index('Metric Value'), h.index('Grid Size')
    agg = collections.OrderedDict()
    tot = 0.0
    for j, r in enumerate(rows[1:]):
        t = float(r[vi].replace(',', '')) / 1000
        n = r[ki][:75]
        if verbose:
            print(f"{j:4d} {t:9.1f} {n[:60]} {r[gi]}")
        a = agg.setdefault(n, [0, 0.0])
        a[0] += 1
        a[1] += t
        tot += t
    for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1])[:25]:
        print(f"{c:4d} {t:9.1f}us {t / tot * 100:5.1f}% {n}")
    print(f"total {tot:.1f} us, {len(rows) - 1} launches")


if __name__ == "__main__":
    main(sys.argv[1], "-v" in sys.argv)
