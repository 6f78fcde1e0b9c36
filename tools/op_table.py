"""Per-op device time (bench.py HIOS_DUMP, sequential instrumented graph)
against each op's roofline: top ops by time (tools/ -- analysis only).

usage: python tools/op_table.py gpurun_out/ops_4096.json [n]
"""
import json
import sys

PEAK_TF, PEAK_GBS = 1645.7, 6554.2


def main():
    d = json.load(open(sys.argv[1]))
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
    tot = sum(o["ms"] for o in d)
    roof_tot = 0.0
    by_kind = {}
    for o in d:
        roof = max(o["gflop"] / PEAK_TF, o["mb"] / PEAK_GBS) * 1e-3 * 1e3  # ms
        o["roof"] = roof
        roof_tot += roof
        k = o["kind"] + ("" if o["kind"] != "conv" else f"{o['k'][0]}x{o['k'][1]}s{o['k'][2]}")
        a = by_kind.setdefault(k, [0, 0.0, 0.0])
        a[0] += 1
        a[1] += o["ms"]
        a[2] += roof
    print(f"total {tot:.3f} ms, roofline {roof_tot:.3f} ms ({roof_tot / tot:.2f})")
    for k, (c, ms, rf) in sorted(by_kind.items(), key=lambda x: -x[1][1]):
        print(f"  {k:14s} n={c:4d} {ms:8.3f} ms  roof {rf:7.3f}  frac {rf / max(ms, 1e-9):.2f}")
    for o in sorted(d, key=lambda o: -o["ms"])[:n]:
        print(f"{o['name'][:28]:28s} {o['kind']:8s} in={o['in'][0] if o['in'] else ''} out={o['shape']} "
              f"k={o['k']} {o['ms'] * 1e3:8.1f} us roof {o['roof'] * 1e3:7.1f} us  "
              f"{o['gflop']:7.2f} GF {o['mb']:7.1f} MB")


if __name__ == "__main__":
    main()
