"""Per-launch rows (kernel, grid, us, DRAM MB) of an ncu --csv launch list, filtered by a substring."""
import csv
import sys


def detail(path, pat, limit=40):
    hdr, cur = None, {}
    out = []
    for r in csv.reader(open(path)):
        if r and r[0] == "ID":
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if pat not in d["Kernel Name"]:
            continue
        key = d["ID"]
        e = cur.setdefault(key, {"k": d["Kernel Name"][:34], "grid": d["Grid Size"]})
        e[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
    for key, e in list(cur.items())[:limit]:
        print(f'{key:>5} {e["k"]:34} {e["grid"]:>14} {e.get("gpu__time_duration.sum", 0) / 1e3:8.1f} us '
              f'rd {e.get("dram__bytes_read.sum", 0) / 1e6:7.2f} MB wr {e.get("dram__bytes_write.sum", 0) / 1e6:7.2f} MB')


if __name__ == "__main__":
    detail(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "", int(sys.argv[3]) if len(sys.argv) > 3 else 40)
