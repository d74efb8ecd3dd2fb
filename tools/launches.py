"""Aggregate an ncu --metrics gpu__time_duration.sum CSV launch list: count and total us per kernel."""
import csv
import sys
from collections import defaultdict


def main(path):
    rows = list(csv.reader(open(path)))
    hdr, agg, order = None, defaultdict(lambda: [0, 0.0]), []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            k = d["Kernel Name"][:70]
            if k not in agg:
                order.append(k)
            agg[k][0] += 1
            agg[k][1] += float(d["Metric Value"].replace(",", "")) / 1e3
    tot = sum(v[1] for v in agg.values()) or 1.0
    for k in order:
        print(f"{agg[k][0]:4d} {agg[k][1]:10.1f} us {100 * agg[k][1] / tot:5.1f}%  {k}")


if __name__ == "__main__":
    main(sys.argv[1])
