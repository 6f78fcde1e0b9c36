"""Time single conv ops through the C-ABI (hios_profile's median of reps =
back-to-back launches of the op's kernel) for a list of Inception-1024 shapes;
optional parity check vs the oracle (--check), fp32 path (--f32).  Kernel
variants are compared as separate builds (tools/build_variant.sh, HIOS_LIB)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen, graphs  # noqa: E402

SHAPES = [  # name, C, K, H, W, kh, kw, s, ph, pw
    ("stem2a", 32, 32, 511, 511, 3, 3, 1, 0, 0),
    ("tiny1x1", 64, 64, 11, 11, 1, 1, 1, 0, 0),     # one tile, one K-step: the fixed cost of a launch
    ("tiny1x1_c256", 256, 64, 11, 11, 1, 1, 1, 0, 0),
    ("4a", 80, 192, 254, 254, 3, 3, 1, 0, 0),
    ("5b_5x5", 48, 64, 125, 125, 5, 5, 1, 2, 2),
    ("5b_1x1", 192, 64, 125, 125, 1, 1, 1, 0, 0),
    ("6a_s2", 288, 384, 125, 125, 3, 3, 2, 0, 0),
    ("6e_1x1", 768, 192, 62, 62, 1, 1, 1, 0, 0),
    ("6e_1x7", 192, 192, 62, 62, 1, 7, 1, 0, 3),
    ("7c_1x1", 2048, 384, 30, 30, 1, 1, 1, 0, 0),
    ("7c_3x3", 448, 384, 30, 30, 3, 3, 1, 1, 1),
    ("7c_1x3", 384, 384, 30, 30, 1, 3, 1, 0, 1),
    ("7c_pool", 2048, 192, 30, 30, 1, 1, 1, 0, 0),
    ("6e_7x1", 192, 192, 62, 62, 7, 1, 1, 3, 0),
    ("7a_s2", 192, 320, 62, 62, 3, 3, 2, 0, 0),
    # Inception-v3 at 4096^2 (compute-heavy)
    ("4a_4096", 80, 192, 1022, 1022, 3, 3, 1, 0, 0),
    ("2a_4096", 32, 32, 2047, 2047, 3, 3, 1, 0, 0),
    ("2b_4096", 32, 64, 2045, 2045, 3, 3, 1, 1, 1),
    ("5b5x5_4096", 48, 64, 509, 509, 5, 5, 1, 2, 2),
    ("7c1x1_4096", 2048, 448, 126, 126, 1, 1, 1, 0, 0),
    ("7b3x3_4096", 448, 384, 126, 126, 3, 3, 1, 1, 1),
    ("5b1x1_4096", 192, 64, 509, 509, 1, 1, 1, 0, 0),
    ("6e1x1_4096", 768, 192, 254, 254, 1, 1, 1, 0, 0),
    ("3b_4096", 64, 80, 1022, 1022, 1, 1, 1, 0, 0),
]


def main():
    check = "--check" in sys.argv
    dtype = "f32" if "--f32" in sys.argv else "bf16"
    only = [a for a in sys.argv[1:] if not a.startswith("--")]
    for (name, C, K, H, W, kh, kw, s, ph, pw) in SHAPES:
        if only and name not in only:
            continue
        g = graphs.GraphSpec("c", C, H, W)
        x0 = g.input()
        g.conv(x0, K, (kh, kw), s=s, p=(ph, pw), relu=1)
        Wt = gen.make_weights(g)
        G = h.hios_graph_create(g.ops, g.edges, C, H, W, dtype, Wt)
        h.hios_profile(G, [0], 30)
        t, _ = h.hios_get_costs(G)
        c, P, Q = h.hios_graph_shape(G, 1)
        fl = 2.0 * K * C * kh * kw * P * Q
        line = f"{name:8s} t={t[1] / 1e3:8.2f}us  {fl / t[1] / 1e3:7.1f} TFLOP/s"
        if check:
            from oracle import infer
            x = gen.make_input(g) - 0.5
            S = h.hios_schedule_lp(G, 1, 1)
            y = h.hios_run(S, x)
            ref = infer.run_graph(g, Wt, x)[1]
            err = float(np.abs(y.reshape(ref.shape) - ref).max() / np.abs(ref).max())
            line += f"  err={err:.2e}"
        print(line, flush=True)


if __name__ == "__main__":
    main()
