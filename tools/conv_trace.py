"""Per-CTA globaltimer timeline of one conv launch (HIOS_TRACE=1)."""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["HIOS_TRACE"] = "1"
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen, graphs  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from conv_micro import SHAPES  # noqa: E402

lib = h.load()
only = sys.argv[1:]
for (name, C, K, H, W, kh, kw, s, ph, pw) in SHAPES:
    if only and name not in only:
        continue
    g = graphs.GraphSpec("c", C, H, W)
    x0 = g.input()
    g.conv(x0, K, (kh, kw), s=s, p=(ph, pw), relu=1)
    Wt = gen.make_weights(g)
    G = h.hios_graph_create(g.ops, g.edges, C, H, W, "bf16", Wt)
    for v in range(2):
        h.hios_set_op_cost(G, v, 1000)
    h.hios_set_edge_cost(G, 0, 1000)
    S = h.hios_schedule_lp(G, 1, 1)
    x = gen.make_input(g)
    for _ in range(3):
        h.hios_run(S, x)
    zero = (ctypes.c_ulonglong * 2048)()
    lib.hios_debug_conv_trace_reset()
    h.hios_run(S, x)
    buf = (ctypes.c_ulonglong * 2048)()
    lib.hios_debug_conv_trace(buf, 2048)
    t = np.array(buf, dtype=np.int64).reshape(256, 8)
    t = t[t[:, 0] > 0]
    t0 = t[:, 0].min()
    rel = (t - t0) / 1e3
    names = ["start", "setup", "tma0", "data0", "mma_end", "epi_in", "epi_out", "exit"]
    print(f"== {name}: {len(t)} CTAs traced, kernel span {rel.max():.2f} us")
    b2 = (ctypes.c_ulonglong * (32 * 48))()
    lib.hios_debug_conv_trace2(b2)
    t2 = (np.array(b2, dtype=np.int64).reshape(32, 3, 16)[0] - t0) / 1e3
    b3 = (ctypes.c_ulonglong * (32 * 8))()
    lib.hios_debug_conv_trace3(b3)
    t3 = (np.array(b3, dtype=np.int64).reshape(32, 8)[0] - t0) / 1e3
    print("   cta0 epi: staged-sync %.2f copied %.2f loop-done %.2f | warps0-1 %.2f 2-3 %.2f 4-5 %.2f 6-7 %.2f" % tuple(t3[:7]))
    b4 = (ctypes.c_ulonglong * (32 * 16))()
    lib.hios_debug_conv_trace4(b4)
    t4 = (np.array(b4, dtype=np.int64).reshape(32, 16) - t0) / 1e3
    lab4 = ["top", "scale", "tfull", "ld0", "ld1", "ld2", "ld3", "ld4", "ld5", "tmem_done", "fence", "bar",
            "tma_issued", "drained"]
    for c in range(min(3, t4.shape[0])):
        print(f"   cta{c} epi4  " + " ".join(f"{n}={v:.2f}" for n, v in zip(lab4, t4[c][:14]) if v > -1e6))
    b5 = (ctypes.c_ulonglong * (32 * 48))()
    lib.hios_debug_conv_trace5(b5)
    t5 = (np.array(b5, dtype=np.int64).reshape(32, 3, 16)[0] - t0) / 1e3
    print("   cta0 epi tfull", " ".join(f"{v:6.2f}" for v in t5[0]))
    print("   cta0 epi done ", " ".join(f"{v:6.2f}" for v in t5[1]))
    print("   cta0 issue   ", " ".join(f"{v:6.2f}" for v in t2[0]))
    print("   cta0 full    ", " ".join(f"{v:6.2f}" for v in t2[1]))
    print("   cta0 emptyok ", " ".join(f"{v:6.2f}" for v in t2[2]))
    for k, n in enumerate(names):
        print(f"   {n:8s} min {rel[:, k].min():7.2f}  med {np.median(rel[:, k]):7.2f}  max {rel[:, k].max():7.2f}")
