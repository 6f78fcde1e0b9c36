"""Summarise ncu --set full reports (one line per launch): duration, SM/DRAM/L2
throughput, tensor-pipe activity, DRAM bytes, occupancy, top stall reason."""
import csv
import io
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "dur_us",
    "dram__bytes_read.sum": "dram_rd",
    "dram__bytes_write.sum": "dram_wr",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed": "mem_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_pct",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed": "tensor_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "occ_pct",
    "launch__grid_size": "grid",
    "launch__registers_per_thread": "regs",
}


def summarise(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        line = {"kernel": d.get("Kernel Name", "")[:60]}
        for k, name in KEYS.items():
            for hk in hdr:
                if hk == k or hk.endswith("." + k) or hk.endswith(k):
                    v = d.get(hk, "")
                    try:
                        line[name] = float(v.replace(",", ""))
                    except ValueError:
                        pass
                    break
        if "dur_us" in line:
            u = units[hdr.index([h for h in hdr if h.endswith("gpu__time_duration.sum")][0])]
            if u == "nsecond":
                line["dur_us"] /= 1e3
            elif u == "msecond":
                line["dur_us"] *= 1e3
        res.append(line)
    return res


if __name__ == "__main__":
    for p in sys.argv[1:]:
        for line in summarise(p):
            print(p.split("/")[-1], line)
