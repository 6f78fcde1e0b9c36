"""Pins for the scheduling oracle (oracle/sched.py) against what PAPER.md and
mathematics fix: the Fig. 4 / Fig. 5 worked examples, closed
forms of the cost model, brute-force optima, brute-force path
enumeration, the Fig. 10 sequential latency."""
import itertools
import json
import os
import random

import pytest

from oracle import sched as S

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def edges_of(d):
    return [tuple(e) for e in d["edges"]]


# ------------------------------------------------------------- Fig. 4
def test_fig4_alg1_every_printed_fact():
    d = load("fig4_alg1.json")
    n, t, E, M = d["n"], d["t"], edges_of(d), d["M"]
    ex = d["expect"]
    assert S.priorities(n, t, E) == ex["priorities"]
    r = S.hios_lp_traced(n, t, E, M, 1, S.group_model(t))
    a1 = r["alg1"]
    assert [p["path"] for p in a1] == [ex["P1"]["ops"], ex["P2"]["ops"], ex["P3"]["ops"]]
    assert a1[0]["gpu"] == ex["P1"]["gpu"]
    assert a1[1]["length"] == ex["P2"]["length"]
    assert a1[1]["trials"] == ex["P2"]["trials"] and a1[1]["gpu"] == ex["P2"]["gpu"]
    assert a1[2]["trials"] == ex["P3"]["trials"] and a1[2]["gpu"] == ex["P3"]["gpu"]
    assert r["L"] == ex["L"]
    # the longer path rejected as invalid at step 2 really is longer (13 vs 11)
    unsched = set(range(n)) - set(ex["P1"]["ops"])
    rej = ex["rejected_longer_invalid"]
    assert S.path_length(rej["ops"], t, E, unsched) == rej["length"]
    assert rej["ops"] not in S.all_valid_paths(n, E, unsched)


def test_fig4_optimal_by_brute_force():
    d = load("fig4_alg1.json")
    n, t, E, M = d["n"], d["t"], edges_of(d), d["M"]
    for w in (1, 2):
        opt, Q, _ = S.brute_force(n, t, E, M, w, S.group_model(t))
        assert opt == d["expect"]["optimal"]
        assert S.validate(n, t, E, Q, w, S.group_model(t)) is None


# ------------------------------------------------------------- Fig. 5
def test_fig5_alg2_trace():
    d = load("fig5_alg2.json")
    n, t, E = d["n"], d["t"], edges_of(d)
    tab = {frozenset(s): c for s, c in d["group_costs"]}
    g = S.table_cost(tab)
    assert S.priorities(n, t, E) == d["expect"]["priorities"]
    Q = [[tuple(s) for s in stl] for stl in d["Q_inter"]]
    assert S.simulate(n, t, E, Q, g)[0] == d["expect"]["L_before"]
    trace = []
    Q2, L2 = S.parallelize(n, t, E, Q, d["w"], g, S.priority_order(n, t, E),
                           S.reachability(n, E), trace)
    assert L2 == d["expect"]["L_after"]
    assert [(v, sorted(W), a, b) for (v, W, a, b) in trace] == \
        [(v, sorted(W), a, b) for (v, W, a, b) in d["expect"]["merges"]]
    assert S.validate(n, t, E, Q2, d["w"], g) is None


# ------------------------------------------------ simulator closed forms
def test_chain_is_sum():
    rng = random.Random(1)
    for _ in range(20):
        n = rng.randint(1, 12)
        t = [rng.randint(1, 50) for _ in range(n)]
        E = [(i, i + 1, rng.randint(0, 30)) for i in range(n - 1)]
        Q, L = S.sequential(n, t, E)
        assert S.simulate(n, t, E, Q, S.group_model(t))[0] == sum(t) == L
        # HIOS-LP on a chain never pays a transfer: one path, one GPU
        Q2, L2, _ = S.hios_lp(n, t, E, 4, 3, S.group_model(t))
        assert L2 == sum(t)


def test_fork_join_closed_form():
    """Source s, branches b_j each on its own GPU, join on s's GPU:
    L = t(s) + max_j(c(s,b_j) + t(b_j) + c(b_j,t)) + t(t), c = 0 on s's GPU."""
    rng = random.Random(2)
    for _ in range(30):
        k = rng.randint(1, 4)
        n = k + 2
        t = [rng.randint(1, 40) for _ in range(n)]
        E = []
        for j in range(1, k + 1):
            E += [(0, j, rng.randint(0, 20)), (j, n - 1, rng.randint(0, 20))]
        Q = [[(0,), (1,), (n - 1,)]] + [[(j,)] for j in range(2, k + 1)]
        L = S.simulate(n, t, E, Q, S.group_model(t))[0]
        best = 0
        for j in range(1, k + 1):
            c1 = E[2 * (j - 1)][2] if j != 1 else 0      # branch 1 shares s's GPU
            c2 = E[2 * (j - 1) + 1][2] if j != 1 else 0
            best = max(best, c1 + t[j] + c2)
        assert L == t[0] + best + t[n - 1]


def test_augmented_dag_longest_path_equals_simulator():
    """Any fixed Q: L = longest path of the augmented DAG (data edges weighted
    t(u,v) across GPUs, 0 on one GPU; stage-order edges 0; node = t(S)).
    Computed here by brute-force path enumeration on small DAGs."""
    rng = random.Random(3)
    for _ in range(40):
        n, t, E = S.random_dag(rng.randint(3, 7), 3, None, 0.8, rng.randint(0, 10**6), unit=10)
        gpu = {v: rng.randrange(2) for v in range(n)}
        order = S.priority_order(n, t, E)
        Q = [[(v,) for v in order if gpu[v] == g] for g in range(2)]
        res = S.simulate(n, t, E, Q, S.group_model(t))
        # augmented graph over ops (singleton stages)
        adj = {v: [] for v in range(n)}
        for (u, v, c) in E:
            adj[u].append((v, c if gpu[u] != gpu[v] else 0))
        for g in range(2):
            for a, b in zip(Q[g], Q[g][1:]):
                adj[a[0]].append((b[0], 0))

        def longest(v):
            return t[v] + max([c + longest(x) for (x, c) in adj[v]] or [0])
        assert res[0] == max(longest(v) for v in range(n))


def test_single_gpu_no_window_is_sequential_sum():
    for seed in range(10):
        n, t, E = S.random_dag(30, 6, None, 0.8, seed, unit=100)
        Q, L, _ = S.hios_lp(n, t, E, 1, 1, S.group_model(t))
        assert L == sum(t)
        assert [s[0] for s in Q[0]] == S.priority_order(n, t, E)


def test_list_schedule_equals_simulator_on_singletons():
    for seed in range(20):
        n, t, E = S.random_dag(25, 5, None, 0.8, seed, unit=100)
        rng = random.Random(seed)
        gpu = {v: rng.randrange(3) for v in range(n)}
        order = S.priority_order(n, t, E)
        L, F, seq = S.list_schedule(n, t, E, gpu, order)
        Q = [[(v,) for v in seq.get(g, [])] for g in range(3)]
        assert S.simulate(n, t, E, Q, S.group_model(t))[0] == L


def test_priority_order_is_topological_and_latest_start():
    for seed in range(10):
        n, t, E = S.random_dag(40, 8, None, 0.8, seed, unit=100)
        order = S.priority_order(n, t, E)
        pos = {v: i for i, v in enumerate(order)}
        assert all(pos[u] < pos[v] for (u, v, _) in E)
        # p(v) = -(latest start time) relative to the critical path length
        p = S.priorities(n, t, E)
        cp = max(p)
        succ, _ = S.succ_lists(n, E)
        for v in range(n):
            latest_finish = min([cp - p[x] - c for (x, c) in succ[v]] or [cp])
            assert cp - p[v] == latest_finish - t[v]


# ------------------------------------------------ longest valid path DP
def test_longest_valid_path_dp_matches_enumeration():
    rng = random.Random(4)
    for _ in range(200):
        n, t, E = S.random_dag(rng.randint(2, 9), rng.randint(2, 4), None, 0.8,
                               rng.randint(0, 10**6), unit=10)
        sched = set(rng.sample(range(n), rng.randint(0, n - 1)))
        unsched = set(range(n)) - sched
        order = S.priority_order(n, t, E)
        rank = {v: i for i, v in enumerate(order)}
        P = S.longest_valid_path(n, t, E, unsched, rank)
        paths = S.all_valid_paths(n, E, unsched)
        best = max(S.path_length(p, t, E, unsched) for p in paths)
        assert S.path_length(P, t, E, unsched) == best
        ties = sorted([[rank[x] for x in p] for p in paths
                       if S.path_length(p, t, E, unsched) == best])
        assert [rank[x] for x in P] == ties[0]


# ---------------------------------------------- HIOS-LP vs brute force
@pytest.mark.parametrize("w", [1, 2])
def test_hios_lp_feasible_and_not_below_optimum(w):
    rng = random.Random(5 + w)
    gaps = []
    for _ in range(40):
        n, t, E = S.random_dag(rng.randint(3, 7), rng.randint(2, 3), None,
                               rng.choice([0.4, 0.8, 1.2]), rng.randint(0, 10**6), unit=10)
        g = S.group_model(t)
        Q, L, _ = S.hios_lp(n, t, E, 2, w, g)
        assert S.validate(n, t, E, Q, w, g) is None
        assert S.simulate(n, t, E, Q, g)[0] == L
        opt, Qo, _ = S.brute_force(n, t, E, 2, w, g)
        assert opt <= L
        gaps.append(L / opt)
    assert min(gaps) == 1.0  # HIOS-LP reaches the optimum on some DAGs


def test_validator_rejects_infeasible():
    d = load("fig5_alg2.json")
    n, t, E = d["n"], d["t"], edges_of(d)
    g = S.group_model(t)
    good = [[(0,), (1,), (3,), (4,), (6,)], [(2,), (5,)]]
    assert S.validate(n, t, E, good, 2, g) is None
    assert "dependent" in S.validate(n, t, E, [[(0, 1), (3,), (4,), (6,)], [(2,), (5,)]], 2, g)
    assert "twice" in S.validate(n, t, E, [[(0,), (1,), (3,), (4,), (6,)], [(2,), (5,), (6,)]], 2, g)
    assert "unscheduled" in S.validate(n, t, E, [[(0,), (1,), (3,), (4,)], [(2,), (5,)]], 2, g)
    # implicit-dependency cycle (C11): GPU0 a, b ; GPU1 x then y ; a->y, x->b
    n2, t2 = 4, [1, 1, 1, 1]
    E2 = [(0, 3, 0), (2, 1, 0)]
    cyc = [[(1,), (0,)], [(3,), (2,)]]
    assert "cycle" in S.validate(n2, t2, E2, cyc, 1, S.group_model(t2))


def test_alg2_cycle_check_blocks_implicit_dependency():
    """C11 example: ops a,b independent in G but merging them deadlocks
    through another GPU's stage order."""
    # GPU0: a(0), b(1); GPU1: x(2) then y(3); edges a->x, y->b
    n, t = 4, [5, 5, 5, 5]
    E = [(0, 2, 0), (3, 1, 0)]
    Q = [[(0,), (1,)], [(3,), (2,)]]
    # order on GPU1 is y then x: merging {a,b} needs y (after x? no) -- check
    g = S.group_model(t)
    merged = [[(0, 1)], [(3,), (2,)]]
    assert S.simulate(n, t, E, merged, g) is not None
    Q = [[(0,), (1,)], [(2,), (3,)]]
    merged = [[(0, 1)], [(2,), (3,)]]
    assert S.simulate(n, t, E, merged, g) is None


def test_fig10_sequential_latency_generator():
    """sequential scheduling of the default random models (200 ops,
    t(v) ~ U[0.1, 4] ms) is 'around 411 ms'; closed form 200 x 2.05 = 410."""
    tot = []
    for seed in range(30):
        n, t, E = S.random_dag(200, 14, None, 0.8, seed, unit=1000)
        assert n == 200 and len(E) == 400
        tot.append(sum(t) / 1000.0)
    mean = sum(tot) / len(tot)
    assert 395 < mean < 425


# ------------------------------------------------------ HIOS-MR (Alg. 3)
def test_mr_diamond_worked_by_hand():
    """Alg. 3 (reading C17) worked by hand on a diamond
    s(1) -> a(4), b(4) -> t(1), every edge 1, M = 2, w = 1.
    Priority order s, a, b, t.  Table (finish times, back-pointer k):
      s: T[0][0]=1
      a: j0: 1+4=5 (k0) | j1: s cross 1+1, +4 = 6 (k0)
      b: j0: k0 -> 5+4=9, k1 (a@1) -> 1+4=5  => 5 (k1)
         j1: k0 (a@0) -> s cross 2, +4 = 6, k1 -> 6+4=10 => 6 (k0)
      t: j0: k0 (b@0,a@1): max(5, a 6+1) + 1 = 8; k1 (b@1,a@0): max(5, 6+1)+1 = 8 -> 8 (first k)
         j1: k0: ready 6, a@1 6, b@0 5+1 -> 7; k1: 7 (tie, first k) -> 7 (k0)
    J = 1; back-track t@1 <- b@0 <- a@1 <- s@0; L = 7 = the optimum (brute force)."""
    t = [1, 4, 4, 1]
    E = [(0, 1, 1), (0, 2, 1), (1, 3, 1), (2, 3, 1)]
    g = S.group_model(t)
    Q, L, gpu = S.hios_mr(4, t, E, 2, 1, g)
    assert gpu == {0: 0, 1: 1, 2: 0, 3: 1}
    assert L == 7 == S.simulate(4, t, E, Q, g)[0]
    assert S.brute_force(4, t, E, 2, 1, g)[0] == 7


def test_mr_chain_and_single_gpu_are_sums():
    rng = random.Random(11)
    for _ in range(20):
        n = rng.randint(1, 10)
        t = [rng.randint(1, 50) for _ in range(n)]
        E = [(i, i + 1, rng.randint(1, 30)) for i in range(n - 1)]
        assert S.hios_mr(n, t, E, 3, 1, S.group_model(t))[1] == sum(t)
    for _ in range(20):
        n, t, E = S.random_dag(rng.randint(2, 12), 3, None, 0.8, rng.randint(0, 10**6), unit=10)
        Q, L, _ = S.hios_mr(n, t, E, 1, 1, S.group_model(t))
        assert L == sum(t) and len(Q) == 1


@pytest.mark.parametrize("w", [1, 2])
def test_mr_feasible_and_not_below_optimum(w):
    rng = random.Random(21 + w)
    for _ in range(30):
        n, t, E = S.random_dag(rng.randint(3, 7), rng.randint(2, 3), None,
                               rng.choice([0.4, 0.8, 1.2]), rng.randint(0, 10**6), unit=10)
        g = S.group_model(t)
        Q, L, _ = S.hios_mr(n, t, E, 2, w, g)
        assert S.validate(n, t, E, Q, w, g) is None
        assert S.simulate(n, t, E, Q, g)[0] == L
        assert S.brute_force(n, t, E, 2, w, g)[0] <= L


# ------------------------------------- IOS comparator (exact, one GPU)
@pytest.mark.parametrize("w", [1, 2, 3])
def test_ios_dp_is_the_single_gpu_optimum(w):
    """P:316 'IOS is an exact algorithm for the optimal schedule in a single
    GPU': the DP equals the brute-force optimum at M = 1, is feasible, and is
    never worse than HIOS-LP at M = 1 (a heuristic over the same space)."""
    rng = random.Random(31 + w)
    for _ in range(40):
        n, t, E = S.random_dag(rng.randint(2, 8), rng.randint(2, 4), None,
                               rng.choice([0.4, 0.8, 1.2]), rng.randint(0, 10**6), unit=10)
        g = S.group_model(t)
        Q, L = S.ios_dp(n, t, E, w, g)
        assert L == S.brute_force(n, t, E, 1, w, g)[0]
        assert S.validate(n, t, E, Q, w, g) is None
        assert S.simulate(n, t, E, Q, g)[0] == L
        assert L <= S.hios_lp(n, t, E, 1, w, g)[1]
        if w == 1:
            assert L == sum(t)


def test_ios_dp_fig5_single_gpu():
    """Fig. 5's graph and group-cost table (pairs the table does not
    list take the C12 model) on one GPU with w = 2: the DP's optimum equals
    brute force and beats running the ops one by one."""
    d = load("fig5_alg2.json")
    n, t, E = d["n"], d["t"], edges_of(d)
    tab = {frozenset(s): c for s, c in d["group_costs"]}
    model = S.group_model(t)

    def g(Sg):
        return tab.get(frozenset(Sg), model(Sg))
    Q, L = S.ios_dp(n, t, E, 2, g)
    assert L == S.brute_force(n, t, E, 1, 2, g)[0]
    assert L < sum(t)
