#!/usr/bin/env python
"""Per-op device times of one schedule (hios_time_ops: each op alone as the
schedule configures it, L2 flushed, CUDA events; and hios_profile's warm t(v))
as JSON, for A/B comparisons of kernel variants (env switches) on one box.

  python tools/op_times.py --model inception_v3 --size 1024 --gpus 1 --window 1 --out gpurun_out/ops_a.json
  python tools/op_times.py --diff gpurun_out/ops_a.json gpurun_out/ops_b.json
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="inception_v3")
    ap.add_argument("--size", type=int, default=1024)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--window", type=int, default=1)
    ap.add_argument("--out", default="")
    ap.add_argument("--diff", nargs=2)
    args = ap.parse_args()
    if args.diff:
        a, b = (json.load(open(p)) for p in args.diff)
        rows = []
        for x, y in zip(a["ops"], b["ops"]):
            if x["cold_us"] > 0:
                rows.append((y["cold_us"] - x["cold_us"], x["name"], x["cold_us"], y["cold_us"], x["warm_us"],
                             y["warm_us"], x["shape"], x["k"]))
        rows.sort()
        print(f"total cold {sum(r[2] for r in rows):.1f} -> {sum(r[3] for r in rows):.1f} us, "
              f"warm {sum(r[4] for r in rows):.1f} -> {sum(r[5] for r in rows):.1f} us")
        for r in rows[:12] + rows[-12:]:
            print(f"{r[0]:+8.2f}  {r[1]:28s} cold {r[2]:8.2f} -> {r[3]:8.2f}  warm {r[4]:8.2f} -> {r[5]:8.2f}  "
                  f"{r[6]} k={r[7]}")
        return
    from paper_conf_cluster_kundus23_b200 import hios as h
    from workloads import gen, graphs
    g = graphs.build(args.model, args.size)
    W = gen.make_weights(g)
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
    h.hios_profile(G, [0], 10)
    tv, _ = h.hios_get_costs(G)
    S = h.hios_schedule_lp(G, args.gpus, args.window)
    cold = h.hios_time_ops(S, 5, 256 << 20)
    ops = [{"id": o.id, "name": o.name, "kind": o.kind, "shape": list(h.hios_graph_shape(G, o.id)),
            "k": [o.kh, o.kw, o.sh, o.sw], "cold_us": float(cold[o.id]) / 1e3, "warm_us": float(tv[o.id]) / 1e3}
           for o in g.ops]
    res = {"model": args.model, "size": args.size, "env": {k: v for k, v in os.environ.items() if k.startswith("HIOS_")},
           "ops": ops}
    print(f"{args.model}@{args.size}: cold sum {sum(o['cold_us'] for o in ops if o['cold_us'] > 0):.1f} us, "
          f"warm sum {sum(o['warm_us'] for o in ops):.1f} us")
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f)


if __name__ == "__main__":
    main()
