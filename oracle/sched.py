"""ORACLE -- test infrastructure only (see oracle/__init__.py).  Step-by-step
reference of the HIOS-LP scheduler (§IV, Alg. 1 + Alg. 2), the cost
model simulator (§III), a feasibility validator and a brute-force
optimal scheduler for tiny DAGs.  Plain Python, integer costs, no blocking or
cleverness beyond what the paper states; the readings of the ambiguous points
are SURVEY.md §8(c) C1-C13 and are listed in DESIGN.md §3.

Graph representation: ``n`` ops 0..n-1, ``t[v]`` = t(v) (int),
``edges`` = list of (u, v, t(u,v)) (parallel edges allowed), ``gcost(S)`` =
t(S) for a frozenset S of >= 2 independent ops.
Schedule Q: list over GPUs of lists of stages; a stage is a tuple of op
ids (order inside a stage is irrelevant).
"""
from __future__ import annotations

import itertools
import random
from typing import Callable, Dict, List, Optional, Sequence, Tuple

INF = float("inf")
Edge = Tuple[int, int, int]


# ----------------------------------------------------------------- helpers
def succ_lists(n, edges):
    s = [[] for _ in range(n)]
    p = [[] for _ in range(n)]
    for (u, v, c) in edges:
        s[u].append((v, c))
        p[v].append((u, c))
    return s, p


def topo_positions(n, edges) -> List[int]:
    """Kahn's algorithm, smallest op id first; position of each op."""
    import heapq
    indeg = [0] * n
    s, _ = succ_lists(n, edges)
    for (_, v, _) in edges:
        indeg[v] += 1
    h = [v for v in range(n) if indeg[v] == 0]
    heapq.heapify(h)
    pos = [-1] * n
    k = 0
    while h:
        v = heapq.heappop(h)
        pos[v] = k
        k += 1
        for (x, _) in s[v]:
            indeg[x] -= 1
            if indeg[x] == 0:
                heapq.heappush(h, x)
    if k != n:
        raise ValueError("graph has a cycle")
    return pos


def reachability(n, edges) -> List[set]:
    """reach[u] = set of ops reachable from u by a directed path (len >= 1)."""
    s, _ = succ_lists(n, edges)
    pos = topo_positions(n, edges)
    order = sorted(range(n), key=lambda v: pos[v])
    reach = [set() for _ in range(n)]
    for u in reversed(order):
        for (v, _) in s[u]:
            reach[u].add(v)
            reach[u] |= reach[v]
    return reach


def independent(a, b, reach) -> bool:
    """C8: no directed path between a and b in G."""
    return a != b and b not in reach[a] and a not in reach[b]


# ------------------------------------------------------- priority (§IV-A)
def priorities(n, t, edges) -> List[int]:
    """p(v) = length (vertex + edge weights) of the longest path from v to the
    last operator of G; p(sink) = t(sink) (C2)."""
    s, _ = succ_lists(n, edges)
    pos = topo_positions(n, edges)
    p = [0] * n
    for v in sorted(range(n), key=lambda v: -pos[v]):
        best = 0
        for (x, c) in s[v]:
            best = max(best, c + p[x])
        p[v] = t[v] + best
    return p


def priority_order(n, t, edges) -> List[int]:
    """Descending p(v); ties -> earlier Kahn position (C2).  A topological order."""
    p = priorities(n, t, edges)
    pos = topo_positions(n, edges)
    return sorted(range(n), key=lambda v: (-p[v], pos[v]))


# -------------------------------------- longest valid path (Alg. 1 line 5)
def path_length(path, t, edges, unsched) -> int:
    """C4: sum of t(v) over the path, the max t(e) between consecutive
    vertices, the max incoming edge from a scheduled op into the first vertex
    and the max outgoing edge from the last vertex to a scheduled op."""
    w = {}
    start = {}
    end = {}
    for (u, v, c) in edges:
        w[(u, v)] = max(w.get((u, v), 0), c)
        if u not in unsched and v in unsched:
            start[v] = max(start.get(v, 0), c)
        if u in unsched and v not in unsched:
            end[u] = max(end.get(u, 0), c)
    L = start.get(path[0], 0) + end.get(path[-1], 0) + sum(t[v] for v in path)
    for a, b in zip(path, path[1:]):
        L += w[(a, b)]
    return L


def longest_valid_path(n, t, edges, unsched: set, rank: Dict[int, int]) -> List[int]:
    """Longest path P in G' = unsched whose intermediate vertices (all but the
    first and the last) have no edge from/to a scheduled vertex (C3),
    length per C4.  Ties: lexicographically smallest sequence of priority
    ranks, a prefix before its extensions.

    Suffix dynamic programme over G' in reverse topological order:
      tail(v) = best path starting at v with v NOT the first vertex
              = max( t(v) + end(v)                       [v last],
                     t(v) + w(v,u) + tail(u).len  (v clean, u in succ(v) & G') )
      full(v) = best path with v first
              = start(v) + max( t(v) + end(v), t(v) + w(v,u) + tail(u).len )
    """
    w: Dict[Tuple[int, int], int] = {}
    start: Dict[int, int] = {}
    end: Dict[int, int] = {}
    clean = {v: True for v in unsched}
    for (u, v, c) in edges:
        if u in unsched and v in unsched:
            w[(u, v)] = max(w.get((u, v), 0), c)
        elif u not in unsched and v in unsched:
            start[v] = max(start.get(v, 0), c)
            clean[v] = False
        elif u in unsched and v not in unsched:
            end[u] = max(end.get(u, 0), c)
            clean[u] = False
    succ: Dict[int, List[int]] = {v: [] for v in unsched}
    for (u, v) in w:
        succ[u].append(v)
    pos = topo_positions(n, edges)
    tail: Dict[int, Tuple[int, List[int]]] = {}

    def better(a, b):  # (len, seq of ranks)
        if a[0] != b[0]:
            return a[0] > b[0]
        return [rank[x] for x in a[1]] < [rank[x] for x in b[1]]

    for v in sorted(unsched, key=lambda v: -pos[v]):
        best = (t[v] + end.get(v, 0), [v])
        if clean[v]:
            for u in succ[v]:
                cand = (t[v] + w[(v, u)] + tail[u][0], [v] + tail[u][1])
                if better(cand, best):
                    best = cand
        tail[v] = best
    overall = None
    for v in unsched:
        best = (start.get(v, 0) + t[v] + end.get(v, 0), [v])
        for u in succ[v]:
            cand = (start.get(v, 0) + t[v] + w[(v, u)] + tail[u][0], [v] + tail[u][1])
            if better(cand, best):
                best = cand
        if overall is None or better(best, overall):
            overall = best
    return overall[1]


def all_valid_paths(n, edges, unsched: set):
    """Brute-force enumeration of every valid path (test pin for the DP)."""
    succ = {v: sorted({b for (a, b, _) in edges if a == v and b in unsched}) for v in unsched}
    clean = {v: all(not ((a == v and b not in unsched) or (b == v and a not in unsched))
                    for (a, b, _) in edges) for v in unsched}
    out = []

    def ext(path):
        out.append(list(path))
        last = path[-1]
        if len(path) > 1 and not clean[last]:
            return  # last is an intermediate candidate only if clean
        for u in succ[last]:
            ext(path + [u])

    for v in unsched:
        ext([v])
    return out


# ------------------------------- temporal list scheduling (Alg. 1 L10-13)
def list_schedule(n, t, edges, gpu: Dict[int, int], order: List[int]):
    """Schedule the mapped vertices in descending-priority order, each at the
    earliest available start on its GPU, appended after the GPU's previous op
    (C1), counting only edges between mapped ops (C5).  Returns (L', F, per-GPU
    op order)."""
    _, preds = succ_lists(n, edges)
    ready: Dict[int, int] = {}
    F: Dict[int, int] = {}
    seq: Dict[int, List[int]] = {}
    for v in order:
        if v not in gpu:
            continue
        g = gpu[v]
        st = ready.get(g, 0)
        for (u, c) in preds[v]:
            if u in gpu:
                st = max(st, F[u] + (c if gpu[u] != g else 0))
        F[v] = st + t[v]
        ready[g] = F[v]
        seq.setdefault(g, []).append(v)
    L = max(F.values()) if F else 0
    return L, F, seq


# --------------------------------------------- simulator (§III)
def stage_cost(S, t, gcost):
    return t[S[0]] if len(S) == 1 else gcost(frozenset(S))


def simulate(n, t, edges, Q, gcost, ops: Optional[set] = None):
    """Event evaluation of schedule Q under the cost model: stages on a GPU run
    sequentially; a stage starts when the previous stage on its GPU finished
    and every input of its ops has arrived: t^S(S') >= t^F(S) + t(u,v) across
    GPUs, >= t^F(S) on the same GPU (Eq. P:100, C16); all ops of a stage start
    together (C13) and the stage lasts t(S).  Returns (L, start, finish)
    keyed by (gpu, stage index), or None if the stage graph has a cycle
    (deadlock)."""
    where = {}
    for g, stl in enumerate(Q):
        for j, S in enumerate(stl):
            for v in S:
                where[v] = (g, j)
    preds: Dict[Tuple[int, int], List[Tuple[Tuple[int, int], int]]] = {}
    for g, stl in enumerate(Q):
        for j in range(len(stl)):
            preds[(g, j)] = [((g, j - 1), 0)] if j > 0 else []
    for (u, v, c) in edges:
        if u not in where or v not in where:
            continue
        su, sv = where[u], where[v]
        if su == sv:
            return None  # dependent ops in one stage: infeasible
        preds[sv].append((su, c if su[0] != sv[0] else 0))
    indeg = {s: len(p) for s, p in preds.items()}
    succ: Dict[Tuple[int, int], List] = {s: [] for s in preds}
    for s, p in preds.items():
        for (x, _) in p:
            succ[x].append(s)
    start, finish = {}, {}
    stack = sorted([s for s, d in indeg.items() if d == 0])
    done = 0
    while stack:
        s = stack.pop()
        st = 0
        for (x, c) in preds[s]:
            st = max(st, finish[x] + c)
        start[s] = st
        finish[s] = st + stage_cost(Q[s[0]][s[1]], t, gcost)
        done += 1
        for y in succ[s]:
            indeg[y] -= 1
            if indeg[y] == 0:
                stack.append(y)
    if done != len(preds):
        return None
    L = max(finish.values()) if finish else 0
    return L, start, finish


# ------------------------------------------------ Alg. 2 (parallelize())
def parallelize(n, t, edges, Q, w, gcost, order, reach, trace=None):
    """Alg. 2 with readings C7-C11: for v_i (i = 1..n-1) in
    priority order, skip it if already grouped (C10); grow a window over the
    next singleton stages on its GPU (sizes 2..w, C7), stop at the first
    dependent pair (C8); merge, reject on a cycle of the scheduled graph (C11),
    reschedule without changing per-GPU order; keep the best window
    and commit only if L' < L (C9)."""
    Q = [list(stl) for stl in Q]
    res = simulate(n, t, edges, Q, gcost)
    assert res is not None
    L = res[0]
    for i in range(n - 1):
        v = order[i]
        g = j = None
        for gg, stl in enumerate(Q):
            for jj, S in enumerate(stl):
                if v in S:
                    g, j = gg, jj
        if len(Q[g][j]) > 1:
            continue
        best_L, best_Q = L, None
        W = [v]
        for p in range(1, w):
            if j + p >= len(Q[g]) or len(Q[g][j + p]) > 1:
                break
            u = Q[g][j + p][0]
            if not all(independent(u, x, reach) for x in W):
                break
            W = W + [u]
            Q2 = [list(stl) for stl in Q]
            Q2[g] = Q2[g][:j] + [tuple(W)] + Q2[g][j + p + 1:]
            r2 = simulate(n, t, edges, Q2, gcost)
            if r2 is None:
                continue
            if r2[0] < best_L:
                best_L, best_Q = r2[0], Q2
        if best_Q is not None:
            if trace is not None:
                trace.append((v, tuple(best_Q[g][j]), L, best_L))
            Q, L = best_Q, best_L
    return Q, L


# ----------------------------------------------------- Alg. 1 (HIOS-LP)
def hios_lp(n, t, edges, M, w, gcost):
    """Alg. 1: iterative longest-valid-path mapping, trial list
    schedules on each GPU (first index wins ties, `L' < L`), then
    Alg. 2 (L17).  Returns (Q, L, gpu_of)."""
    r = hios_lp_traced(n, t, edges, M, w, gcost)
    return r["Q"], r["L"], r["gpu"]


def hios_lp_traced(n, t, edges, M, w, gcost):
    """hios_lp with the Alg. 1 path trace and the Alg. 2 merge trace."""
    order = priority_order(n, t, edges)
    rank = {v: i for i, v in enumerate(order)}
    reach = reachability(n, edges)
    unsched = set(range(n))
    gpu: Dict[int, int] = {}
    alg1 = []
    while unsched:
        P = longest_valid_path(n, t, edges, unsched, rank)
        length = path_length(P, t, edges, unsched)
        unsched -= set(P)
        best_L, best_i, trials = INF, None, []
        for i in range(M):
            trial = dict(gpu)
            trial.update({v: i for v in P})
            L2, _, _ = list_schedule(n, t, edges, trial, order)
            trials.append(L2)
            if L2 < best_L:
                best_L, best_i = L2, i
        gpu.update({v: best_i for v in P})
        alg1.append({"path": P, "length": length, "trials": trials, "gpu": best_i})
    _, _, seq = list_schedule(n, t, edges, gpu, order)
    Q0 = [[(v,) for v in seq.get(g, [])] for g in range(M)]
    L0 = simulate(n, t, edges, Q0, gcost)[0]
    alg2 = []
    Q, L = parallelize(n, t, edges, Q0, w, gcost, order, reach, alg2)
    return {"Q": Q, "L": L, "gpu": gpu, "Q_inter": Q0, "L_inter": L0,
            "alg1": alg1, "alg2": alg2, "order": order}


def sequential(n, t, edges):
    """Sequential scheduling baseline: one GPU, priority order."""
    order = priority_order(n, t, edges)
    return [[(v,) for v in order]], sum(t)


# --------------------------------------------------- validator (C6)
def validate(n, t, edges, Q, w, gcost) -> Optional[str]:
    """Feasibility per P:86-100 / C6.  Returns None if feasible, else a reason."""
    reach = reachability(n, edges)
    seen = {}
    for g, stl in enumerate(Q):
        for j, S in enumerate(stl):
            if not 1 <= len(S) <= max(w, 1):
                return f"stage {g},{j} has {len(S)} ops > w={w}"
            for a, b in itertools.combinations(S, 2):
                if not independent(a, b, reach):
                    return f"stage {g},{j}: ops {a},{b} dependent"
            for v in S:
                if v in seen:
                    return f"op {v} scheduled twice"
                seen[v] = (g, j)
    if len(seen) != n:
        return f"{n - len(seen)} ops unscheduled"
    res = simulate(n, t, edges, Q, gcost)
    if res is None:
        return "stage graph has a cycle (deadlock)"
    L, start, finish = res
    for (u, v, c) in edges:
        su, sv = seen[u], seen[v]
        need = c if su[0] != sv[0] else 0
        if start[sv] - finish[su] < need:
            return f"edge {u}->{v} violates Eq. P:100"
    for g, stl in enumerate(Q):
        for j in range(1, len(stl)):
            if start[(g, j)] < finish[(g, j - 1)]:
                return f"stages {g},{j - 1} and {g},{j} overlap"
    return None


# ------------------------------------------- brute-force optimum (tiny)
def brute_force(n, t, edges, M, w, gcost):
    """Exact optimum of P:94-100 over every GPU mapping (restricted growth:
    GPUs are homogeneous) x every per-GPU ordered partition into stages
    of <= w pairwise-independent ops; each candidate is evaluated with the same
    simulator.  Exponential: for <= 8-9 ops."""
    reach = reachability(n, edges)
    _, preds = succ_lists(n, edges)
    best = [INF, None]

    def per_gpu_orders(ops_g: List[int]):
        res = []
        opset = set(ops_g)

        def rec(placed: set, seq):
            if len(placed) == len(ops_g):
                res.append(list(seq))
                return
            rem = [v for v in ops_g if v not in placed]
            avail = [v for v in rem if all(u in placed or u not in opset for (u, _) in preds[v])]
            for k in range(1, min(w, len(avail)) + 1):
                for A in itertools.combinations(avail, k):
                    if all(independent(a, b, reach) for a, b in itertools.combinations(A, 2)):
                        seq.append(tuple(A))
                        rec(placed | set(A), seq)
                        seq.pop()

        rec(set(), [])
        return res

    def mappings(i, cur, mx):
        if i == n:
            yield list(cur)
            return
        for g in range(min(mx + 2, M)):
            cur.append(g)
            yield from mappings(i + 1, cur, max(mx, g))
            cur.pop()

    count = 0
    for mp in mappings(0, [], -1):
        per = []
        for g in range(M):
            per.append(per_gpu_orders([v for v in range(n) if mp[v] == g]))
        for combo in itertools.product(*per):
            Q = [list(c) for c in combo]
            r = simulate(n, t, edges, Q, gcost)
            if r is None:
                continue
            count += 1
            if r[0] < best[0]:
                best = [r[0], Q]
    return best[0], best[1], count


# ----------------------------------------------- group-cost models
def group_model(t, num=7, den=10):
    """C12 synthetic t(S) = max(max t(v), floor(sum t(v) * num / den)) -- a
    documented model for cost-only tests (parity unpinned against hardware)."""
    def gcost(S):
        return max(max(t[v] for v in S), (sum(t[v] for v in S) * num) // den)
    return gcost


def table_cost(table: Dict[frozenset, int]):
    def gcost(S):
        return table[frozenset(S)]
    return gcost


# --------------------------------------- random DAG generator (§V-A)
def random_dag(n_ops=200, n_layers=14, n_deps=None, p=0.8, seed=0, unit=1000):
    """n_ops operators in n_layers layers, 2*n_ops dependencies, t(v)
    uniform in [0.1, 4] ms, transfer time max(0.1 ms, p * t(v)) (C18).  Costs
    are integers in 1/unit ms (default microseconds).  Edges go from a lower
    layer to a higher one; every op past layer 0 gets a predecessor in the
    previous layer."""
    rng = random.Random(seed)
    n_deps = 2 * n_ops if n_deps is None else n_deps
    n_layers = max(1, min(n_layers, n_ops))
    cuts = sorted(rng.sample(range(1, n_ops), n_layers - 1))
    bounds = [0] + cuts + [n_ops]
    layer = []
    for li in range(n_layers):
        layer += [li] * (bounds[li + 1] - bounds[li])
    t = [rng.randint(int(0.1 * unit), int(4 * unit)) for _ in range(n_ops)]
    es = set()
    for v in range(n_ops):
        li = layer[v]
        if li > 0:
            u = rng.randrange(bounds[li - 1], bounds[li])
            es.add((u, v))
    tries = 0
    while len(es) < n_deps and tries < 100 * n_deps:
        tries += 1
        u, v = rng.randrange(n_ops), rng.randrange(n_ops)
        if layer[u] < layer[v]:
            es.add((u, v))
    edges = [(u, v, max(int(0.1 * unit), int(round(p * t[u])))) for (u, v) in sorted(es)]
    return n_ops, t, edges


# ------------------------------------------------ Alg. 3 (HIOS-MR)
def hios_mr(n, t, edges, M, w, gcost):
    """Alg. 3 (the extracted pseudo-code is garbled, reconstruction
    C17): an n x M table (t_{i,j}, g_{i,j}) over the ops in priority order;
    t_{i,j} = earliest finish of v_i on GPU j given the recorded schedule of
    v_1..v_{i-1} that ends with v_{i-1} on GPU k (k chosen to minimise it,
    first k wins ties: `if t_{i,j} > t_k + t(v_i)`); v_1 on GPU 1; back-track
    from J = argmin_j t_{n,j}; then Alg. 2.  Returns (Q, L, gpu_of)."""
    order = priority_order(n, t, edges)
    pos = {v: i for i, v in enumerate(order)}
    _, preds = succ_lists(n, edges)
    INFV = float("inf")
    T = [[INFV] * M for _ in range(n)]
    Gb = [[0] * M for _ in range(n)]
    T[0][0] = t[order[0]]
    for i in range(1, n):
        vi = order[i]
        for j in range(min(M, i + 1)):
            for k in range(min(M, i)):
                if T[i - 1][k] == INFV:
                    continue
                # schedule of v_1..v_{i-1} recorded with v_{i-1} on GPU k (L10-12)
                tF, gp = {}, {}
                m = k
                for l in range(i - 1, -1, -1):
                    tF[order[l]] = T[l][m]
                    gp[order[l]] = m
                    m = Gb[l][m]
                # L14: GPU j becomes free after the last op recorded on it
                tk = max([tF[order[l]] for l in range(i) if gp[order[l]] == j] or [0])
                # L15-19: inputs of v_i
                for (u, c) in preds[vi]:
                    if pos[u] >= i:
                        continue
                    tk = max(tk, tF[u] if gp[u] == j else tF[u] + c)
                if T[i][j] > tk + t[vi]:  # L20-21
                    T[i][j] = tk + t[vi]
                    Gb[i][j] = k
    J = min(range(M), key=lambda j: (T[n - 1][j], j))  # L22
    gpu = {}
    m = J
    for i in range(n - 1, -1, -1):  # L24-25
        gpu[order[i]] = m
        m = Gb[i][m]
    Q = [[(v,) for v in order if gpu[v] == g] for g in range(M)]
    reach = reachability(n, edges)
    Q, L = parallelize(n, t, edges, Q, w, gcost, order, reach)  # L27
    return Q, L, gpu


# ------------------------------------- exact single-GPU optimum ("IOS")
def ios_dp(n, t, edges, w, gcost):
    """The IOS comparator ("an exact algorithm for the
    optimal schedule in a single GPU", dynamic programming): on one GPU, the
    sequence of stages -- sets of <= w pairwise-independent ops whose inputs
    are all produced by earlier stages -- minimising L = sum t(S) (P:86-100 at
    M = 1).  Plain DP over the set D of finished ops (always downward closed):
        f(V) = 0,  f(D) = min over E of t(E) + f(D | E),
    E ranging over the independent subsets of ready(D) of size 1..w,
    enumerated in itertools.combinations order of the ready ops sorted by id,
    sizes ascending, first strict minimum kept.  Exponential; for small
    graphs.  Returns (Q, L) with Q = [[stage, ...]] on GPU 0."""
    reach = reachability(n, edges)
    _, preds = succ_lists(n, edges)
    pset = [set(u for (u, _) in preds[v]) for v in range(n)]
    full = frozenset(range(n))
    memo: Dict[frozenset, Tuple[int, Optional[tuple]]] = {full: (0, None)}

    def cost(E):
        return t[E[0]] if len(E) == 1 else gcost(frozenset(E))

    def f(D: frozenset):
        if D in memo:
            return memo[D][0]
        ready = sorted(v for v in range(n) if v not in D and pset[v] <= D)
        best, arg = INF, None
        for k in range(1, min(w, len(ready)) + 1):
            for E in itertools.combinations(ready, k):
                if any(not independent(a, b, reach) for a, b in itertools.combinations(E, 2)):
                    continue
                c = cost(E) + f(D | frozenset(E))
                if c < best:
                    best, arg = c, E
        memo[D] = (best, arg)
        return best

    L = f(frozenset())
    stages, D = [], frozenset()
    while D != full:
        E = memo[D][1]
        stages.append(tuple(E))
        D = D | frozenset(E)
    return [stages], L
