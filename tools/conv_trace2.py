"""Per-tile globaltimer timeline of CTA 0 of one conv launch (HIOS_TRACE=1):
halo/producer issue, MMA start/end, epilogue tfull/stores-issued, for the
first 16 tiles (tools/ -- analysis only).

usage: python tools/conv_trace2.py [op_micro conv name ...]
"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["HIOS_TRACE"] = "1"
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from op_micro import SHAPES, build  # noqa: E402

lib = h.load()
only = sys.argv[1:]
for (name, kind, C, H, W, prm) in SHAPES:
    if kind != "conv" or (only and name not in only):
        continue
    g = build(kind, C, H, W, prm)
    G = h.hios_graph_create(g.ops, g.edges, C, H, W, "bf16", gen.make_weights(g))
    for v in range(g.n_ops):
        h.hios_set_op_cost(G, v, 1000)
    for e in range(len(g.edges)):
        h.hios_set_edge_cost(G, e, 1000)
    S = h.hios_schedule_lp(G, 1, 1)
    x = gen.make_input(g)
    for _ in range(3):
        h.hios_run(S, x)
    lib.hios_debug_conv_trace_reset()
    h.hios_run(S, x)
    b = (ctypes.c_ulonglong * 2048)()
    lib.hios_debug_conv_trace(b, 2048)
    t = np.array(b, dtype=np.int64).reshape(256, 8)
    t = t[t[:, 0] > 0]
    t0 = t[:, 0].min()
    b2 = (ctypes.c_ulonglong * (32 * 48))()
    lib.hios_debug_conv_trace2(b2)
    t2 = (np.array(b2, dtype=np.int64).reshape(32, 3, 16)[0] - t0) / 1e3
    b5 = (ctypes.c_ulonglong * (32 * 48))()
    lib.hios_debug_conv_trace5(b5)
    t5 = (np.array(b5, dtype=np.int64).reshape(32, 3, 16)[0] - t0) / 1e3
    print(f"== {name}: kernel span {((t.max() - t0) / 1e3):.2f} us, CTA0 setup {(t[0,1]-t0)/1e3:.2f}")
    print("   tile  prod_issue  mma_start  mma_end  epi_tfull  epi_stored")
    for k in range(16):
        print(f"   {k:4d}  " + "  ".join(f"{v:9.2f}" for v in (t2[0][k], t2[1][k], t2[2][k], t5[0][k], t5[1][k])))
