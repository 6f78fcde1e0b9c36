"""Summarise an ncu --csv launch list (gpu__time_duration.sum [+ dram bytes])
per kernel name: launches, total / mean time, share, DRAM bytes."""
import collections
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    ids = collections.OrderedDict()
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            e = ids.setdefault(d["ID"], {"name": d["Kernel Name"], "grid": d["Grid Size"],
                                         "block": d["Block Size"]})
            try:
                e[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
            except ValueError:
                pass
    return list(ids.values())


def short(n):
    n = n.replace("void ", "").replace("hios::", "")
    return n.split("(")[0][:48]


def main(path):
    L = load(path)
    tot = collections.OrderedDict()
    for e in L:
        t = tot.setdefault(short(e["name"]), [0, 0.0, 0.0])
        t[0] += 1
        t[1] += e.get("gpu__time_duration.sum", 0.0)
        t[2] += e.get("dram__bytes_read.sum", 0.0) + e.get("dram__bytes_write.sum", 0.0)
    T = sum(v[1] for v in tot.values())
    print(f"{'kernel':48s} {'launch':>6s} {'total_us':>9s} {'mean_us':>8s} {'share':>6s} {'dram_MB':>8s}")
    for k, v in sorted(tot.items(), key=lambda x: -x[1][1]):
        print(f"{k:48s} {v[0]:6d} {v[1] / 1e3:9.1f} {v[1] / 1e3 / v[0]:8.2f} {v[1] / T:6.3f} {v[2] / 1e6:8.1f}")
    print(f"total {T / 1e3:.1f} us over {len(L)} launches")


if __name__ == "__main__":
    main(sys.argv[1])
