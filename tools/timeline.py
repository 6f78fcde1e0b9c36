#!/usr/bin/env python
"""Diagnostic (not a bench number): the kernel timeline of one HIOS schedule's
CUDA-graph replay, traced with torch.profiler (CUPTI activity records: every
kernel's start/end and stream, concurrency preserved).  Reports, per step:
the step span, the summed kernel busy time, the union of busy intervals, and
the idle gaps on the critical chain -- i.e. how much of the latency is kernel
execution vs launch/dependency latency between kernels.

  python tools/timeline.py --model inception_v3 --size 1024 --window 5 --out gpurun_out/tl.json
"""
from __future__ import annotations

import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="inception_v3")
    ap.add_argument("--size", type=int, default=1024)
    ap.add_argument("--window", type=int, default=5)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/timeline.json")
    args = ap.parse_args()
    import torch
    from torch.profiler import ProfilerActivity, profile

    from paper_conf_cluster_kundus23_b200 import hios as h
    from workloads import gen, graphs
    g = graphs.build(args.model, args.size)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
    h.hios_profile(G, [0], 5)
    res = {}
    for name, (M, w) in {"hios_lp": (args.gpus, args.window), "sequential": (1, 1)}.items():
        S = h.hios_schedule_lp(G, M, w)
        d_in = torch.from_numpy(x).cuda()
        d_out = torch.empty(h.hios_output_numel(S), device="cuda")
        st = torch.cuda.current_stream()
        flush = torch.empty(64 * 1024 * 1024, device="cuda")
        for _ in range(5):
            h.hios_run_device(S, d_in.data_ptr(), d_out.data_ptr(), st.cuda_stream)
        torch.cuda.synchronize()
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            for i in range(args.steps):
                flush.fill_(float(i))
                torch.cuda.synchronize()
                h.hios_run_device(S, d_in.data_ptr(), d_out.data_ptr(), st.cuda_stream)
                torch.cuda.synchronize()
        evs = [e for e in prof.events() if e.device_type.name == "CUDA"]
        kern = []
        for e in evs:
            nm = e.name
            if "fill" in nm.lower() and "Fill" in nm:
                continue
            kern.append((e.time_range.start, e.time_range.end, nm))
        kern.sort()
        # split into steps at gaps > 200 us
        steps, cur = [], []
        for k in kern:
            if cur and k[0] - max(c[1] for c in cur) > 200:
                steps.append(cur)
                cur = []
            cur.append(k)
        if cur:
            steps.append(cur)
        out = []
        for s in steps:
            t0 = min(a for a, _, _ in s)
            t1 = max(b for _, b, _ in s)
            busy = sum(b - a for a, b, _ in s)
            iv = sorted((a, b) for a, b, _ in s)
            union, ca, cb = 0.0, None, None
            for a, b in iv:
                if ca is None or a > cb:
                    if ca is not None:
                        union += cb - ca
                    ca, cb = a, b
                else:
                    cb = max(cb, b)
            union += (cb - ca) if ca is not None else 0
            by = {}
            for a, b, nm in s:
                key = nm.split("<")[0].split("(")[0]
                d = by.setdefault(key, [0, 0.0])
                d[0] += 1
                d[1] += b - a
            out.append({"span_us": t1 - t0, "busy_us": busy, "union_us": union, "n": len(s),
                        "by_kernel": {k: {"n": v[0], "us": v[1]} for k, v in sorted(by.items(), key=lambda kv: -kv[1][1])},
                        "kernels": [(a - t0, b - t0, nm[:60]) for a, b, nm in s]})
        res[name] = out
        print(name, [(round(o["span_us"], 1), round(o["union_us"], 1), round(o["busy_us"], 1), o["n"]) for o in out])
        if out:
            last = out[-1]
            print("  by kernel:", {k: (v["n"], round(v["us"], 1)) for k, v in list(last["by_kernel"].items())[:8]})
    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(res, f)


if __name__ == "__main__":
    main()
