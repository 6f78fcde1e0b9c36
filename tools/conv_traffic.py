"""DRAM traffic per conv_tc launch from an ncu launch list (CSV of
gpu__time_duration.sum, dram__bytes_read.sum, dram__bytes_write.sum; ncu's
default cache control flushes caches between replays, so this is the cold
traffic) -> profiles/conv_traffic_<workload>.json, read by bench.py for the
roofline "traffic" field.  usage: python tools/conv_traffic.py launches.csv workload
"""
import csv
import json
import os
import sys


def main():
    path, workload = sys.argv[1], sys.argv[2]
    rows = list(csv.reader(open(path)))
    hdr = None
    per = {}
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if "conv_tc_kernel" not in d["Kernel Name"]:
            continue
        v = float(d["Metric Value"].replace(",", ""))
        unit = d.get("Metric Unit", "")
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "usecond": 1e3}.get(unit, 1)
        per.setdefault(d["ID"], {})[d["Metric Name"]] = v * scale
    launches = [m for m in per.values() if "dram__bytes_read.sum" in m]
    tot = sum(m["dram__bytes_read.sum"] + m.get("dram__bytes_write.sum", 0) for m in launches)
    out = {"workload": workload, "launches": len(launches), "bytes_per_launch": tot / max(len(launches), 1),
           "source": os.path.basename(path) + " (ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,"
                     "dram__bytes_write.sum --clock-control none, cold caches)"}
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    # on the GPU box only gpurun_out/ comes back: write there, copy to profiles/ here
    dst = os.path.join(root, sys.argv[3] if len(sys.argv) > 3 else "profiles", f"conv_traffic_{workload}.json")
    json.dump(out, open(dst, "w"), indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
