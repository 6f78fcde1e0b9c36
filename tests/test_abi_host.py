"""Host-side tests of the C-ABI library (no GPU): the library loads and exports
every symbol include/hios.h declares; graph validation; the C++ HIOS-LP
scheduler and simulator are bit-identical to the step-by-step CPU oracle on
the same integer costs (Fig. 4 / Fig. 5 fixtures, random DAGs, the benchmark
DAGs with synthetic costs)."""
import ctypes
import json
import os
import random
import re

import numpy as np
import pytest

from oracle import sched as S
from paper_conf_cluster_kundus23_b200 import hios
from workloads import gen, graphs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "hios.h")).read()
    names = set(re.findall(r"\b(hios_[a-z_0-9]+)\s*\(", hdr))
    names -= {"hios_op", "hios_edge"}
    assert len(names) >= 25
    lib = ctypes.CDLL(hios.LIB_PATH)
    missing = [n for n in sorted(names) if not hasattr(lib, n)]
    assert not missing, missing
    assert hios.hios_abi_version() == 1


class _Op:
    def __init__(self, kind="identity", **kw):
        self.kind = kind
        self.__dict__.update(kw)


def _cost_graph(n, t, edges, dtype="f32"):
    """A graph whose structure is (n, edges) built from identity ops on a tiny
    tensor (host-only: shapes are valid, costs injected)."""
    indeg = [0] * n
    for (u, v, _) in edges:
        indeg[v] += 1
    # one input op feeding every source; identity ops elsewhere; add ops for joins
    ops = []
    slots = [0] * n
    E = []
    for v in range(n):
        k = "add" if indeg[v] > 1 else ("identity" if indeg[v] == 1 else "identity")
        ops.append(_Op(k, id=v, out_c=8, cost_ns=t[v]))
    # a zero-cost input op n feeding each source
    src_ops = [v for v in range(n) if indeg[v] == 0]
    ops.append(_Op("input", id=n, out_c=8, cost_ns=0))
    for (u, v, c) in edges:
        E.append((u, v, slots[v], c))
        slots[v] += 1
    for v in src_ops:
        E.append((n, v, 0, 0))
    # sinks: join them into one op so the graph has a unique sink
    outdeg = [0] * (n + 1)
    for (u, v, _, _) in E:
        outdeg[u] += 1
    sinks = [v for v in range(n) if outdeg[v] == 0]
    if len(sinks) > 1:
        ops.append(_Op("add", id=n + 1, out_c=8, cost_ns=0))
        for i, v in enumerate(sinks):
            E.append((v, n + 1, i, 0))
    G = hios.hios_graph_create(ops, [(a, b, s) for (a, b, s, _) in E], 8, 4, 4, dtype,
                               edge_costs=[c for (_, _, _, c) in E])
    t_all = list(t) + [0] + ([0] if len(sinks) > 1 else [])
    E_all = [(a, b, c) for (a, b, _, c) in E]
    return G, len(ops), t_all, E_all


def _oracle_Q(Q):
    return [[tuple(sorted(s)) for s in q] for q in Q]


@pytest.mark.parametrize("w", [1, 2, 3])
@pytest.mark.parametrize("M", [1, 2, 4])
def test_scheduler_bit_exact_vs_oracle_random(M, w):
    rng = random.Random(100 * M + w)
    for it in range(25):
        n0 = rng.randint(3, 40)
        n, t, E = S.random_dag(n0, rng.randint(2, 8), None, rng.choice([0.4, 0.8, 1.2]),
                               rng.randint(0, 10**6), unit=1000)
        G, N, t_all, E_all = _cost_graph(n, t, E)
        hios.hios_set_group_model(G, 7, 10)
        s = hios.hios_schedule_lp(G, M, w)
        Qo, Lo, _ = S.hios_lp(N, t_all, E_all, M, w, S.group_model(t_all))
        assert hios.hios_schedule_latency_ns(s) == Lo
        assert hios.stages_to_Q(s) == _oracle_Q(Qo)


def test_scheduler_fig4_fig5_through_abi():
    d = json.load(open(os.path.join(ROOT, "tests", "golden", "fig4_alg1.json")))
    G, N, t_all, E_all = _cost_graph(d["n"], d["t"], [tuple(e) for e in d["edges"]])
    hios.hios_set_group_model(G, 7, 10)
    s = hios.hios_schedule_lp(G, 2, 1)
    assert hios.hios_schedule_latency_ns(s) == d["expect"]["L"] == 16
    # F5: import the inter-GPU schedule, then Alg. 2 via hios_schedule_lp is not
    # reachable with the paper's table; check the simulator on the imported Q
    d5 = json.load(open(os.path.join(ROOT, "tests", "golden", "fig5_alg2.json")))
    G5, N5, t5, E5 = _cost_graph(d5["n"], d5["t"], [tuple(e) for e in d5["edges"]])
    for ops, c in d5["group_costs"]:
        hios.hios_set_group_cost(G5, ops, c)
    gpu = [0] * N5
    st = [0] * N5
    for gi, q in enumerate(d5["Q_inter"]):
        for j, stage in enumerate(q):
            for v in stage:
                gpu[v], st[v] = gi, j + (1 if gi == 0 else 0)
    # the helper's input op (id n) goes first on GPU 0; the sink-join op last
    gpu[d5["n"]], st[d5["n"]] = 0, 0
    if N5 > d5["n"] + 1:
        gpu[N5 - 1], st[N5 - 1] = 0, len(d5["Q_inter"][0]) + 1
    s5 = hios.hios_schedule_import(G5, 2, 2, gpu, st)
    assert hios.hios_schedule_latency_ns(s5) == 18
    # merged version (the final schedule of Fig. 5): 16
    st2 = list(st)
    for v in (3,):        # v4 joins v2's stage
        st2[v] = st[1]
    for v in (6,):        # v7 joins v5's stage
        st2[v] = st[4]
    # renumber GPU-0 stages densely
    used = sorted({st2[v] for v in range(N5) if gpu[v] == 0})
    ren = {x: i for i, x in enumerate(used)}
    for v in range(N5):
        if gpu[v] == 0:
            st2[v] = ren[st2[v]]
    s6 = hios.hios_schedule_import(G5, 2, 2, gpu, st2)
    assert hios.hios_schedule_latency_ns(s6) == 16


def test_benchmark_dags_bit_exact_with_synthetic_costs():
    """Inception-v3 / SqueezeNet / RandWire / NASNet DAGs, synthetic integer
    costs, M in {1, 2, 4, 8}, w in {1, 3}: C++ == oracle."""
    rng = random.Random(7)
    for name, size in [("inception_v3", 299), ("squeezenet", 224), ("randwire_ws", 224),
                       ("nasnet_a_large", 331)]:
        g = graphs.build(name, size)
        for op in g.ops:
            op.cost_ns = 0 if op.kind == "input" else rng.randint(2000, 90000)
        ec = [rng.randint(1000, 60000) for _ in g.edges]
        W = gen.make_weights(g)
        G = hios.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W, edge_costs=ec)
        hios.hios_set_group_model(G, 7, 10)
        t = [op.cost_ns for op in g.ops]
        E = [(s, d, c) for (s, d, _), c in zip(g.edges, ec)]
        for M, w in [(1, 1), (1, 3), (2, 3), (8, 3)] if name != "nasnet_a_large" else [(2, 2)]:
            s = hios.hios_schedule_lp(G, M, w)
            Qo, Lo, _ = S.hios_lp(g.n_ops, t, E, M, w, S.group_model(t))
            assert hios.hios_schedule_latency_ns(s) == Lo, (name, M, w)
            assert hios.stages_to_Q(s) == _oracle_Q(Qo), (name, M, w)
            assert S.validate(g.n_ops, t, E, Qo, w, S.group_model(t)) is None


def test_shape_inference_matches_oracle():
    from oracle import infer
    for name, size in [("inception_v3", 299), ("squeezenet", 224), ("randwire_ws", 96),
                       ("nasnet_a_large", 96), ("tiny", None)]:
        g = graphs.build(name, size)
        W = gen.make_weights(g)
        G = hios.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
        out = infer.run_graph(g, W, gen.make_input(g))
        for op in g.ops:
            assert hios.hios_graph_shape(G, op.id) == out[op.id].shape, (name, op.name)


def test_graph_validation_errors():
    ops = [_Op("input", id=0, out_c=8), _Op("identity", id=1), _Op("identity", id=2)]
    with pytest.raises(hios.HiosError) as e:
        hios.hios_graph_create(ops, [(0, 1, 0), (1, 2, 0), (2, 1, 0)], 8, 4, 4, "f32")
    assert e.value.code in (1, 2)
    with pytest.raises(hios.HiosError) as e:   # cycle, slots well-formed
        ops4 = [_Op("input", id=0, out_c=8), _Op("add", id=1), _Op("identity", id=2), _Op("identity", id=3)]
        hios.hios_graph_create(ops4, [(0, 1, 0), (2, 1, 1), (1, 2, 0), (1, 3, 0)], 8, 4, 4, "f32")
    assert e.value.code == 2
    with pytest.raises(hios.HiosError) as e:   # shape mismatch: conv in_c
        w = {1: {"weight": np.zeros((4, 3, 1, 1), np.float32)}}
        hios.hios_graph_create([_Op("input", id=0, out_c=8), _Op("conv", id=1, in_c=3, out_c=4, kh=1, kw=1,
                                                                  sh=1, sw=1)],
                               [(0, 1, 0)], 8, 4, 4, "f32", w)
    assert e.value.code == 3
    with pytest.raises(hios.HiosError):        # self loop
        hios.hios_graph_create([_Op("input", id=0, out_c=8), _Op("identity", id=1)],
                               [(0, 1, 0), (1, 1, 1)], 8, 4, 4, "f32")


def test_missing_costs_is_state_error():
    g = graphs.tiny(8, 8, 8)
    G = hios.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "f32", gen.make_weights(g))
    with pytest.raises(hios.HiosError) as e:
        hios.hios_schedule_lp(G, 2, 2)
    assert e.value.code == 8


def test_executor_queries_and_stage_modes_host_rules():
    """Host-side rules of the executor queries (no GPU): the stage mode
    accepts STREAMS / GROUPED / DATAFLOW / AUTO and rejects others
    (HIOS_E_INVALID); the mode used, the conv tile plan and the hoisted-ReLU
    flag exist only after a run (HIOS_E_STATE); bad op ids are HIOS_E_INVALID."""
    g = graphs.tiny(8, 8, 8)
    G = hios.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", gen.make_weights(g))
    for op in g.ops:
        hios.hios_set_op_cost(G, op.id, 1000)
    for e in range(g.n_edges):
        hios.hios_set_edge_cost(G, e, 100)
    hios.hios_set_group_model(G, 7, 10)
    for mode in ("streams", "grouped", "dataflow", "auto"):
        S = hios.hios_schedule_lp(G, 1, 2)
        hios.hios_schedule_stage_mode(S, mode)
    S = hios.hios_schedule_lp(G, 1, 2)
    with pytest.raises(hios.HiosError) as e:
        hios.hios_schedule_stage_mode(S, 7)
    assert e.value.code == 1
    with pytest.raises(hios.HiosError) as e:
        hios.hios_schedule_stage_mode_used(S)
    assert e.value.code == 8
    with pytest.raises(hios.HiosError) as e:
        hios.hios_op_plan(S, 1)
    assert e.value.code == 8
    with pytest.raises(hios.HiosError) as e:
        hios.hios_op_output_relu(S, 1)
    assert e.value.code == 8
    with pytest.raises(hios.HiosError) as e:
        hios.hios_op_output_relu(S, g.n_ops)
    assert e.value.code == 1


def test_import_rejects_infeasible():
    n, t, E = 4, [5, 5, 5, 5], [(0, 2, 0), (3, 1, 0)]
    G, N, t_all, E_all = _cost_graph(n, t, E)
    hios.hios_set_group_model(G, 7, 10)
    inp = N - 2 if N == 6 else N - 1
    # GPU0: a, b ; GPU1: x then y, edges a->x, y->b ; merging {a,b} deadlocks (C11)
    gpu = [0, 0, 1, 1] + [0] * (N - 4)
    st = [1, 1, 0, 1] + [0] * (N - 4)
    if N == 6:
        st[5] = 2
    with pytest.raises(hios.HiosError) as e:
        hios.hios_schedule_import(G, 2, 2, gpu, st)
    assert e.value.code == 2
    with pytest.raises(hios.HiosError) as e:   # window exceeded
        hios.hios_schedule_import(G, 2, 1, gpu, st)
    assert e.value.code == 1


@pytest.mark.parametrize("M,w", [(1, 1), (2, 1), (2, 2), (4, 3)])
def test_hios_mr_bit_exact_vs_oracle(M, w):
    """Alg. 3 (HIOS-MR): C++ == step-by-step oracle."""
    rng = random.Random(900 + 10 * M + w)
    for _ in range(15):
        n, t, E = S.random_dag(rng.randint(3, 30), rng.randint(2, 6), None, rng.choice([0.4, 0.8]),
                               rng.randint(0, 10**6), unit=1000)
        G, N, t_all, E_all = _cost_graph(n, t, E)
        hios.hios_set_group_model(G, 7, 10)
        s = hios.hios_schedule_mr(G, M, w)
        Qo, Lo, _ = S.hios_mr(N, t_all, E_all, M, w, S.group_model(t_all))
        assert hios.hios_schedule_latency_ns(s) == Lo
        assert hios.stages_to_Q(s) == _oracle_Q(Qo)
        assert S.validate(N, t_all, E_all, Qo, w, S.group_model(t_all)) is None


def test_simulation_study_orderings():
    """§V-style cost-model study (200 ops, 14 layers, 400 deps,
    4 GPUs, t(v) ~ U[0.1, 4] ms, transfer max(0.1 ms, 0.8 t(v))) through the
    C-ABI: HIOS-LP beats sequential and the IOS-style single-GPU schedule and is
    on average no worse than HIOS-MR.  The generator's layer
    structure and t(S) are not given in the paper (C12), so only orderings are
    asserted; the ratios are recorded in DESIGN.md."""
    res = {"seq": [], "ios": [], "mr": [], "lp": [], "lp_inter": []}
    for seed in range(8):
        n, t, E = S.random_dag(200, 14, None, 0.8, seed, unit=1000)
        G, N, t_all, E_all = _cost_graph(n, t, E)
        hios.hios_set_group_model(G, 9, 10)
        res["seq"].append(hios.hios_schedule_latency_ns(hios.hios_schedule_lp(G, 1, 1)))
        res["ios"].append(hios.hios_schedule_latency_ns(hios.hios_schedule_lp(G, 1, 3)))
        res["mr"].append(hios.hios_schedule_latency_ns(hios.hios_schedule_mr(G, 4, 3)))
        res["lp"].append(hios.hios_schedule_latency_ns(hios.hios_schedule_lp(G, 4, 3)))
        res["lp_inter"].append(hios.hios_schedule_latency_ns(hios.hios_schedule_lp(G, 4, 1)))
    m = {k: sum(v) / len(v) for k, v in res.items()}
    assert m["lp"] < m["ios"] < m["seq"]
    assert m["lp"] <= m["mr"]
    assert m["lp"] <= m["lp_inter"]          # Alg. 2 never makes Alg. 1's schedule worse
    assert 350e3 < m["seq"] / 1.0 < 470e3     # ~411 ms sequential (Fig. 10)


def test_group_cost_sources():
    """hios_group_cost: t(v) for singletons, injected t(S) first, else the
    group model; no source -> HIOS_E_STATE; bad ids -> HIOS_E_INVALID."""
    n, t, E = S.random_dag(6, 2, None, 0.8, 3, unit=1000)
    G, N, t_all, E_all = _cost_graph(n, t, E)
    assert hios.hios_group_cost(G, [1]) == t_all[1]
    with pytest.raises(hios.HiosError):
        hios.hios_group_cost(G, [1, 2])          # nothing known yet
    hios.hios_set_group_cost(G, [2, 1], 12345)
    assert hios.hios_group_cost(G, [1, 2]) == 12345
    hios.hios_set_group_model(G, 7, 10)
    assert hios.hios_group_cost(G, [1, 2]) == 12345  # injected wins
    assert hios.hios_group_cost(G, [1, 3]) == S.group_model(t_all)((1, 3))
    for bad in ([1, 1], [N + 5], []):
        with pytest.raises(hios.HiosError):
            hios.hios_group_cost(G, bad)


@pytest.mark.parametrize("w", [1, 2, 3])
def test_ios_latency_equals_oracle_dp(w):
    """hios_schedule_ios (C++ DP, cut-vertex decomposition) reaches the same
    optimum L as the oracle's plain DP (ties may pick different stages, so
    the schedule is checked for feasibility, not equality)."""
    rng = random.Random(70 + w)
    for _ in range(30):
        n, t, E = S.random_dag(rng.randint(2, 9), rng.randint(2, 4), None, 0.8, rng.randint(0, 10**6), unit=1000)
        G, N, t_all, E_all = _cost_graph(n, t, E)
        hios.hios_set_group_model(G, 7, 10)
        s = hios.hios_schedule_ios(G, w)
        Qo, Lo = S.ios_dp(N, t_all, E_all, w, S.group_model(t_all))
        assert hios.hios_schedule_latency_ns(s) == Lo
        Q = hios.stages_to_Q(s)
        assert S.validate(N, t_all, E_all, Q, w, S.group_model(t_all)) is None


def test_ios_on_benchmark_dags_not_worse_than_hios_m1():
    for name, size in [("inception_v3", 299), ("squeezenet", 224), ("randwire_ws", 224)]:
        g = graphs.build(name, size)
        G = hios.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", gen.make_weights(g))
        for op in g.ops:
            hios.hios_set_op_cost(G, op.id, 1000 + (37 * op.id) % 500)
        for e in range(g.n_edges):
            hios.hios_set_edge_cost(G, e, 100)
        hios.hios_set_group_model(G, 7, 10)
        L_ios = hios.hios_schedule_latency_ns(hios.hios_schedule_ios(G, 4))
        assert L_ios <= hios.hios_schedule_latency_ns(hios.hios_schedule_lp(G, 1, 4))


def test_simulation_study_trends():
    """Figs. 7, 10, 11 trends through the C-ABI on the
    §V generator (4 seeds; tools/sim_study.py runs the full sweeps): HIOS-LP's
    speedup over sequential grows with the number of GPUs and beats HIOS-MR
    from 4 GPUs on; HIOS-LP latency falls as the layer count falls (more
    parallelism); its speedup falls as the transfer/compute ratio p grows.
    (Magnitudes differ from the paper's: its generator is underspecified, C18,
    DESIGN.md §10.)"""
    def mean_lat(M=4, layers=14, p=0.8, kind="lp", seeds=4):
        tot = 0
        for seed in range(seeds):
            n, t, E = S.random_dag(200, layers, None, p, seed, unit=1000)
            G, N, t_all, E_all = _cost_graph(n, t, E)
            hios.hios_set_group_model(G, 9, 10)
            if kind == "seq":
                s = hios.hios_schedule_lp(G, 1, 1)
            elif kind == "mr":
                s = hios.hios_schedule_mr(G, M, 3)
            else:
                s = hios.hios_schedule_lp(G, M, 3)
            tot += hios.hios_schedule_latency_ns(s)
        return tot / seeds
    seq = mean_lat(kind="seq")
    sp = [seq / mean_lat(M=m) for m in (2, 4, 8)]
    assert sp[0] < sp[1] < sp[2]                                    # Fig. 7
    assert mean_lat(M=4) < mean_lat(M=4, kind="mr")                # Fig. 7/8: LP beats MR
    assert mean_lat(M=8) < mean_lat(M=8, kind="mr")
    assert mean_lat(layers=6) < mean_lat(layers=14) < mean_lat(layers=22)   # Fig. 10
    assert mean_lat(p=0.4, seeds=12) < mean_lat(p=1.2, seeds=12)   # Fig. 11
