"""Time the stride-2 small-C stem convs (Inception/RandWire 3x3 3->32,
SqueezeNet 7x7 3->96) alone through the C-ABI (hios_profile's t(v), which
includes the s2d staging kernel when the s2d path is taken); --check adds
parity vs the oracle.  Compare the tensor-core s2d path with the direct
CUDA-core kernel as two builds (tools/build_variant.sh, HIOS_LIB=ab/libhios_<name>.so)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen, graphs  # noqa: E402

SHAPES = [  # name, C, K, H, W, k, s, p
    ("incep1a@1024", 3, 32, 1024, 1024, 3, 2, 0),
    ("incep1a@2048", 3, 32, 2048, 2048, 3, 2, 0),
    ("incep1a@4096", 3, 32, 4096, 4096, 3, 2, 0),
    ("rw_stem@2048", 3, 39, 2048, 2048, 3, 2, 1),
    ("squeeze1@2048", 3, 96, 2048, 2048, 7, 2, 0),
]


def main():
    check = "--check" in sys.argv
    for (name, C, K, H, W, k, s, p) in SHAPES:
        g = graphs.GraphSpec("c", C, H, W)
        x0 = g.input()
        g.conv(x0, K, (k, k), s=s, p=(p, p), relu=1)
        Wt = gen.make_weights(g)
        G = h.hios_graph_create(g.ops, g.edges, C, H, W, "bf16", Wt)
        h.hios_profile(G, [0], 30)
        t, _ = h.hios_get_costs(G)
        line = f"{name:14s} t={t[1] / 1e3:8.2f}us"
        if check and H <= 1024:
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
