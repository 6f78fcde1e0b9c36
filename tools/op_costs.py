"""Profiled t(v) of every op and t(S) of every stage of the HIOS-LP schedule,
against each op's roofline (tools/ -- analysis only).

usage: python tools/op_costs.py [model] [size] [window]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen, graphs  # noqa: E402

PEAK_TF, PEAK_GBS = 1645.7, 6554.2


def main():
    model = sys.argv[1] if len(sys.argv) > 1 else "inception_v3"
    size = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
    w = int(sys.argv[3]) if len(sys.argv) > 3 else 4
    g = graphs.build(model, size)
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", gen.make_weights(g))
    h.hios_profile(G, [0], 20)
    S = h.hios_schedule_lp(G, 1, w)
    t, _ = h.hios_get_costs(G)
    shapes = [h.hios_graph_shape(G, v) for v in range(len(g.ops))]
    rows = []
    for o in g.ops:
        v = o.id
        c, P, Q = shapes[v]
        fl, by = 0.0, 0.0
        ins = [shapes[u] for u in g.preds(v)]
        if o.kind == "conv":
            ci, H, W = ins[0]
            fl = 2.0 * c * ci * o.kh * o.kw * P * Q
            by = 2.0 * (ci * H * W + c * ci * o.kh * o.kw + c * P * Q)
        elif o.kind in ("maxpool", "avgpool", "gap", "add", "linear", "sepconv"):
            by = 2.0 * (sum(a * b * d for a, b, d in ins) + c * P * Q)
        roof = max(fl / PEAK_TF / 1e6, by / PEAK_GBS / 1e3)  # us
        rows.append((t[v] / 1e3, roof, o.name, o.kind, (c, P, Q)))
    print(f"sum t(v) {sum(r[0] for r in rows):.1f} us, sum roof {sum(r[1] for r in rows):.1f} us")
    by_kind = {}
    for r in rows:
        k = by_kind.setdefault(r[3], [0, 0.0, 0.0])
        k[0] += 1
        k[1] += r[0]
        k[2] += r[1]
    for k, (n, tt, rr) in sorted(by_kind.items(), key=lambda x: -x[1][1]):
        print(f"  {k:8s} n={n:3d} t={tt:8.1f} us roof={rr:7.1f} us")
    print("top ops by t(v):")
    for r in sorted(rows, reverse=True)[:25]:
        print(f"  {r[0]:8.2f} us (roof {r[1]:6.2f})  {r[2]:32s} {r[3]:8s} {r[4]}")
    Q = h.stages_to_Q(S)[0]
    print(f"stages {len(Q)}; predicted L = {h.hios_schedule_latency_ns(S) / 1e3:.1f} us")
    tot = 0
    for k, St in enumerate(Q):
        ts = h.hios_group_cost(G, list(St)) / 1e3
        tot += ts
        names = ",".join(g.ops[v].name.replace("Mixed_", "M").replace("branch", "b") for v in St)
        print(f"  S{k:02d} t(S)={ts:7.2f} us  sum t(v)={sum(t[v] for v in St) / 1e3:7.2f}  {names}")
    print(f"sum t(S) {tot:.1f} us")


if __name__ == "__main__":
    main()
