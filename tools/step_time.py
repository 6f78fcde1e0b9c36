#!/usr/bin/env python
"""Device time of one schedule's step (hios_run_device, CUDA events, L2 flushed
between steps) for A/B runs against another build of the library (HIOS_LIB):
uses only ABI calls that exist since round 1.

  python tools/step_time.py --model inception_v3 --size 1024 --window 5
"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="inception_v3")
    ap.add_argument("--size", type=int, default=1024)
    ap.add_argument("--windows", default="1,5")
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--stage-mode", default="streams")
    args = ap.parse_args()
    import torch
    from paper_conf_cluster_kundus23_b200 import hios as h
    from workloads import gen, graphs
    g = graphs.build(args.model, args.size)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
    h.hios_profile(G, [0], 10)
    d_in = torch.from_numpy(x).cuda()
    st = torch.cuda.current_stream()
    flush = torch.empty(64 << 20, device="cuda")
    out = []
    for w in [int(v) for v in args.windows.split(",")]:
        S = h.hios_schedule_lp(G, 1, w)
        if args.stage_mode != "streams":
            h.hios_schedule_stage_mode(S, args.stage_mode)
        d_out = torch.empty(h.hios_output_numel(S), device="cuda")
        for _ in range(5):
            h.hios_run_device(S, d_in.data_ptr(), d_out.data_ptr(), st.cuda_stream)
        ts = []
        for i in range(args.steps):
            flush.fill_(float(i))
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(st)
            h.hios_run_device(S, d_in.data_ptr(), d_out.data_ptr(), st.cuda_stream)
            b.record(st)
            ts.append((a, b))
        torch.cuda.synchronize()
        ms = [a.elapsed_time(b) for a, b in ts]
        out.append(f"w={w}: {np.mean(ms):.4f} ms (median {np.median(ms):.4f}, predicted "
                   f"{h.hios_schedule_latency_ns(S) / 1e6:.4f})")
    print(f"{args.model}@{args.size} lib={os.environ.get('HIOS_LIB', 'in-tree')} mode={args.stage_mode}: " + "; ".join(out),
          flush=True)


if __name__ == "__main__":
    main()
