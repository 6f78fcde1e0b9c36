"""Fig. 1 analog on B200: latency ratio
between parallel and sequential execution of two identical convolutions
(5x5, stride 1, 48 input channels -> 48 output channels, 'same' padding) for
input sizes 8^2 ... 4096^2.

Both numbers come from the framework's own profiler through the C-ABI:
  sequential = t(A) + t(B)            (hios_profile: each op alone)
  parallel   = t({A, B})              (hios_group_cost: forked onto two
                                       streams of one GPU and joined)
ratio = parallel / sequential; < 1 means running the two ops concurrently on
one GPU pays (the paper's crossover on an A40 is between 64^2 and 128^2).

Fig. 2 analog: ratio of the transfer time of the conv's input to its
compute time.  With one GPU visible the transfer cannot cross NVLink, so two
columns are given: the profiler's t(u, v) of the input edge measured on this
device (a device-local peer-store push + flag release/acquire), and the
NVLink model bytes / 770 GB/s (the measured B200 peer-copy bandwidth of
B200_PROFILING.md, not measured here).

usage: python tools/fig1_contention.py [--dtypes bf16,f32] [--out path.json]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen, graphs  # noqa: E402


def pair_graph(hw: int):
    g = graphs.GraphSpec("fig1", 48, hw, hw)
    x = g.input()
    a = g.conv(x, 48, (5, 5), s=1, p=(2, 2), relu=1, name="convA")
    b = g.conv(x, 48, (5, 5), s=1, p=(2, 2), relu=1, name="convB")
    g.concat([a, b], name="cat")
    return g, a, b


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dtypes", default="bf16,f32")
    ap.add_argument("--sizes", default="8,16,32,64,128,256,512,1024,2048,4096")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    rows = []
    for dt in args.dtypes.split(","):
        for hw in [int(s) for s in args.sizes.split(",")]:
            g, a, b = pair_graph(hw)
            G = h.hios_graph_create(g.ops, g.edges, 48, hw, hw, dt, gen.make_weights(g))
            h.hios_profile(G, [0], args.reps)
            t, te = h.hios_get_costs(G)
            seq = int(t[a] + t[b])
            in_bytes = 48 * hw * hw * (2 if dt == "bf16" else 4)
            e_in = [i for i, (u, v, _) in enumerate(g.edges) if v == a][0]
            par = h.hios_group_cost(G, [a, b])
            fl = 2.0 * 48 * 48 * 25 * hw * hw
            r = {"dtype": dt, "hw": hw, "t_a_us": t[a] / 1e3, "t_b_us": t[b] / 1e3,
                 "seq_us": seq / 1e3, "par_us": par / 1e3, "ratio_par_over_seq": par / seq,
                 "tflops_alone": fl / t[a] / 1e3,
                 "fig2_input_bytes": in_bytes, "fig2_t_edge_local_us": te[e_in] / 1e3,
                 "fig2_t_nvlink_model_us": in_bytes / 770e9 * 1e6,
                 "fig2_ratio_local": te[e_in] / t[a], "fig2_ratio_nvlink_model": in_bytes / 770e9 * 1e9 / t[a]}
            rows.append(r)
            print(f"{dt:5s} {hw:5d}^2  t(A) {r['t_a_us']:9.2f} us  t(B) {r['t_b_us']:9.2f} us  "
                  f"t(A||B) {r['par_us']:9.2f} us  ratio {r['ratio_par_over_seq']:.3f}  "
                  f"({r['tflops_alone']:.1f} TFLOP/s alone)  fig2 xfer/compute local {r['fig2_ratio_local']:.2f} "
                  f"nvlink-model {r['fig2_ratio_nvlink_model']:.3f}", flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump({"what": "Fig. 1 analog (P:62): two 5x5 48->48 convs, parallel/sequential",
                       "rows": rows}, f, indent=1)


if __name__ == "__main__":
    main()
