"""Host logic of the cross-GPU transports (no GPU needed).

* The NCCL transport posts every process's sends / receives in one global
  order (hios_schedule_transfers; csrc/nccl.cpp transfer_order).  Two
  properties make that safe, checked here on random DAG schedules for
  M = 2..8 against the schedule itself (hios_schedule_stages):
  - capture-time consistency: when GPU l posts its communication actions up
    to the receive a stage needs, every send among them has a producer in an
    earlier stage of l (the executor raises HIOS_E_STATE otherwise);
  - deadlock freedom: a discrete simulation of rendezvous semantics (a send
    and its receive complete together, each communication stream executes its
    actions strictly in order, a stage runs after the previous stage of its
    GPU and after the receives of its remote inputs) always completes.
* Transport selection through the C-ABI: codes, and the state rules (before
  the first run; NCCL init needs rank mode).
"""
import random

import pytest

from oracle import sched as OS
from paper_conf_cluster_kundus23_b200 import hios
from test_abi_host import _cost_graph


def _schedule(seed, M, w):
    rng = random.Random(seed)
    n0 = rng.randint(5, 40)
    n, t, E = OS.random_dag(n0, rng.randint(2, 8), None, rng.choice([0.2, 0.5, 1.0]), rng.randint(0, 10**6),
                            unit=1000)
    G, N, t_all, E_all = _cost_graph(n, t, E)
    hios.hios_set_group_model(G, 7, 10)
    S = hios.hios_schedule_lp(G, M, w)
    return G, S, N, E_all


def _check_order(S, N, E_all, M):
    og, ost, nst = hios.hios_schedule_stages(S)
    og, ost = og.tolist(), ost.tolist()
    xfers = hios.hios_schedule_transfers(S)
    # exactly the (producer, consumer GPU) pairs of cross-GPU edges, once each
    pairs = {(u, og[v]) for (u, v, _) in E_all if og[u] != og[v]}
    assert sorted(xfers) == sorted(pairs) and len(set(xfers)) == len(xfers)
    stages = {g: [[v for v in range(N) if og[v] == g and ost[v] == j] for j in range(int(nst[g]))]
              for g in range(M)}
    acts = {g: [k for k, (u, d) in enumerate(xfers) if og[u] == g or d == g] for g in range(M)}
    # capture-time consistency (exec.cu enqueue_stage_program: post())
    for g in range(M):
        nxt, done_ops = 0, set()
        for S_ in stages[g]:
            need = [k for k, (u, d) in enumerate(xfers)
                    if d == g and any(og[v] == g and ost[v] == ost[S_[0]] for (uu, v, _) in E_all if uu == u)]
            for k in need:
                i = acts[g].index(k)
                for kk in acts[g][nxt:i + 1]:
                    u, d = xfers[kk]
                    if og[u] == g:
                        assert u in done_ops, f"GPU {g} would post the send of op {u} before running it"
                nxt = max(nxt, i + 1)
            done_ops.update(S_)
    # rendezvous simulation
    head = {g: 0 for g in range(M)}
    nxt_stage = {g: 0 for g in range(M)}
    done_x, done_ops = set(), set()
    remote_in = {}
    for (u, v, _) in E_all:
        if og[u] != og[v]:
            remote_in.setdefault(v, set()).add(xfers.index((u, og[v])))
    progress = True
    while progress:
        progress = False
        for g in range(M):
            while nxt_stage[g] < len(stages[g]):
                S_ = stages[g][nxt_stage[g]]
                if all(remote_in.get(v, set()) <= done_x for v in S_):
                    done_ops.update(S_)
                    nxt_stage[g] += 1
                    progress = True
                else:
                    break
        for g in range(M):
            if head[g] >= len(acts[g]):
                continue
            k = acts[g][head[g]]
            u, d = xfers[k]
            src = og[u]
            peer = d if src == g else src
            if head[peer] < len(acts[peer]) and acts[peer][head[peer]] == k and u in done_ops:
                head[g] += 1
                head[peer] += 1
                done_x.add(k)
                progress = True
    assert all(nxt_stage[g] == len(stages[g]) for g in range(M)), "deadlock: stages left"
    assert all(head[g] == len(acts[g]) for g in range(M)), "deadlock: transfers left"
    return len(xfers)


@pytest.mark.parametrize("M", [2, 3, 4, 8])
def test_nccl_transfer_order_consistent_and_deadlock_free(M):
    total = 0
    for seed in range(40):
        G, S, N, E_all = _schedule(1000 * M + seed, M, random.Random(seed).choice([1, 2, 3]))
        total += _check_order(S, N, E_all, M)
    assert total > 0  # the random schedules do use several GPUs


def test_transfer_order_benchmark_dags():
    from workloads import gen, graphs
    rng = random.Random(5)
    for name, size in [("inception_v3", 299), ("randwire_ws", 224), ("nasnet_a_large", 331)]:
        g = graphs.build(name, size)
        G = hios.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", gen.make_weights(g))
        for op in g.ops:
            hios.hios_set_op_cost(G, op.id, 0 if op.kind == "input" else rng.randint(1000, 50000))
        for e in range(g.n_edges):
            hios.hios_set_edge_cost(G, e, rng.randint(100, 5000))
        hios.hios_set_group_model(G, 7, 10)
        for M in (2, 4, 8):
            S = hios.hios_schedule_lp(G, M, 3)
            E_all = [(u, v, 0) for (u, v, _) in g.edges]
            _check_order(S, g.n_ops, E_all, M)


def test_transport_selection_rules():
    G, S, N, E_all = _schedule(7, 2, 2)
    for t in ("peer", "copy", "nccl", 0, 1, 2):
        hios.hios_schedule_transport(S, t)
    with pytest.raises(hios.HiosError) as ei:
        hios.hios_schedule_transport(S, 3)
    assert ei.value.code == 1
    # NCCL init outside rank mode is a state error (no device work)
    hios.hios_schedule_transport(S, "nccl")
    with pytest.raises(hios.HiosError) as ei:
        hios.hios_schedule_nccl_init(S, bytes(128), 2, 0)
    assert ei.value.code == 8
