"""Summarise an ncu --csv launch list (gpu__time_duration + dram bytes per launch) by kernel."""
import collections
import csv
import sys


def table(path, top=40):
    hdr, agg = None, collections.defaultdict(lambda: [0, 0.0, 0.0, 0.0])
    for r in csv.reader(open(path)):
        if r and r[0] == "ID":
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        k, m = d["Kernel Name"][:60], d["Metric Name"]
        v = float(d["Metric Value"].replace(",", ""))
        if m == "gpu__time_duration.sum":
            agg[k][0] += 1
            agg[k][1] += v
        elif m == "dram__bytes_read.sum":
            agg[k][2] += v
        elif m == "dram__bytes_write.sum":
            agg[k][3] += v
    tot = sum(a[1] for a in agg.values())
    print("| kernel | launches | mean us | share | DRAM read MB/launch | DRAM write MB/launch |")
    print("|---|---|---|---|---|---|")
    for k, (n, t, rd, wr) in sorted(agg.items(), key=lambda x: -x[1][1])[:top]:
        print(f"| {k} | {n} | {t / n / 1e3:.1f} | {100 * t / tot:.1f}% | {rd / n / 1e6:.2f} | {wr / n / 1e6:.2f} |")


if __name__ == "__main__":
    table(sys.argv[1])
