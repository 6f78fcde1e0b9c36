"""Time single ops through the C-ABI (hios_profile: median of back-to-back
in-graph replays of the op's kernels) for the heaviest shapes of the benchmark
DAGs (gpurun_out/ops_*.json); env switches (HIOS_POOL_OLD, HIOS_DW_OLD,
...; A/B variants are separate builds, HIOS_LIB=ab/libhios_<name>.so) select kernel variants.

usage: python tools/op_micro.py [name ...]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen, graphs  # noqa: E402

PEAK_TF, PEAK_GBS = 1645.7, 6554.2

# name, kind, C, H, W, params
SHAPES = [
    ("i4096_maxpool1", "maxpool", 64, 2045, 2045, dict(k=3, s=2, p=0)),
    ("i4096_maxpool2", "maxpool", 192, 1020, 1020, dict(k=3, s=2, p=0)),
    ("i4096_6a_maxpool", "maxpool", 288, 509, 509, dict(k=3, s=2, p=0)),
    ("i4096_avgpool5d", "avgpool", 288, 509, 509, dict(k=3, s=1, p=1)),
    ("i4096_avgpool6b", "avgpool", 768, 254, 254, dict(k=3, s=1, p=1)),
    ("sq_maxpool2", "maxpool", 96, 1021, 1021, dict(k=3, s=2, p=0, ceil=1)),
    ("sq_maxpool6", "maxpool", 256, 510, 510, dict(k=3, s=2, p=0, ceil=1)),
    ("nas_avg_s1", "avgpool", 168, 256, 256, dict(k=3, s=1, p=1, cip=0)),
    ("nas_sep7s2_stem", "sepconv", 42, 1023, 1023, dict(k=7, s=2, K=42, reps=2)),
    ("nas_sep5_cell0", "sepconv", 168, 256, 256, dict(k=5, s=1, K=168, reps=2)),
    ("nas_sep7s2_red0", "sepconv", 336, 256, 256, dict(k=7, s=2, K=336, reps=2)),
    ("rw_sep3_n5", "sepconv", 78, 256, 256, dict(k=3, s=1, K=78, reps=1, n_in=4)),
    ("sq_conv1", "conv", 3, 2048, 2048, dict(K=96, k=7, s=2, p=0)),
    ("rw_conv1", "conv", 3, 2048, 2048, dict(K=39, k=3, s=2, p=1)),
    ("rw_conv2", "conv", 39, 1024, 1024, dict(K=78, k=3, s=2, p=1)),
    ("i4096_conv1a", "conv", 3, 4096, 4096, dict(K=32, k=3, s=2, p=0)),
    ("i4096_conv5d1x1", "conv", 288, 509, 509, dict(K=64, k=1, s=1, p=0)),
    ("i4096_conv7c1x1", "conv", 2048, 126, 126, dict(K=384, k=1, s=1, p=0)),
    ("i4096_conv2a", "conv", 32, 2047, 2047, dict(K=32, k=3, s=1, p=0)),
    ("i4096_conv2b", "conv", 32, 2045, 2045, dict(K=64, k=3, s=1, p=1)),
    ("i4096_conv4a", "conv", 80, 1022, 1022, dict(K=192, k=3, s=1, p=0)),
    ("i4096_conv3b", "conv", 64, 1022, 1022, dict(K=80, k=1, s=1, p=0)),
    ("i4096_6a", "conv", 288, 509, 509, dict(K=384, k=3, s=2, p=0)),
]


def build(kind, C, H, W, prm):
    g = graphs.GraphSpec("m", C, H, W)
    x0 = g.input()
    if kind == "maxpool":
        g.maxpool(x0, prm["k"], prm["s"], prm["p"], ceil_mode=prm.get("ceil", 0))
    elif kind == "avgpool":
        g.avgpool(x0, prm["k"], prm["s"], prm["p"], count_include_pad=prm.get("cip", 1))
    elif kind == "sepconv":
        n_in = prm.get("n_in", 1)
        ins = [x0] if n_in == 1 else [g.conv(x0, C, 1, relu=0) for _ in range(n_in)]
        g.sepconv(ins, prm["K"], prm["k"], s=prm["s"], reps=prm["reps"])
    elif kind == "conv":
        g.conv(x0, prm["K"], prm["k"], s=prm["s"], p=prm["p"])
    return g


def main():
    only = [a for a in sys.argv[1:] if not a.startswith("--")]
    esz = 2
    for (name, kind, C, H, W, prm) in SHAPES:
        if only and not any(name.startswith(o) for o in only):
            continue
        g = build(kind, C, H, W, prm)
        G = h.hios_graph_create(g.ops, g.edges, C, H, W, "bf16", gen.make_weights(g))
        h.hios_profile(G, [0], 20)
        t, _ = h.hios_get_costs(G)
        v = g.n_ops - 1
        c, P, Q = h.hios_graph_shape(G, v)
        ci, hi, wi = h.hios_graph_shape(G, g.preds(v)[0])
        by = (ci * hi * wi * len(g.preds(v)) + c * P * Q) * esz
        fl = 0.0
        if kind == "conv":
            fl = 2.0 * prm["K"] * ci * prm["k"] ** 2 * P * Q
        roof = max(fl / PEAK_TF / 1e12, by / PEAK_GBS / 1e9) * 1e6
        print(f"{name:18s} t={t[v] / 1e3:9.2f} us  roof {roof:8.2f} us  frac {roof / (t[v] / 1e3):.2f}  "
              f"({by / (t[v]) :.0f} GB/s, {fl / t[v] / 1e3:.0f} TFLOP/s)", flush=True)


if __name__ == "__main__":
    main()
