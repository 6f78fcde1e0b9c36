// sched.cpp -- host-side HIOS-LP scheduler (§IV).
//
//   priorities       p(v), §IV-A
//   longest path     Alg. 1 line 5, readings C3/C4
//   list schedule    Alg. 1 lines 10-13, readings C1/C5
//   hios_lp          Alg. 1 lines 1-16
//   parallelize      Alg. 2, readings C7-C11
//   simulate         cost model of §III: stage start = max(prev
//                    stage on the GPU, inputs' finish + t(u,v) across GPUs)
//
// Integer nanosecond costs; every tie rule is fixed so the
// result is bit-identical to the step-by-step CPU oracle on the same costs.
#include <algorithm>
#include <limits>

#include <functional>
#include <unordered_map>
#include "internal.h"

namespace hios {

int64_t Graph::stage_cost(const std::vector<int>& S_in) {
  if (S_in.size() == 1) return op_cost(S_in[0]);
  std::vector<int> S = S_in;
  std::sort(S.begin(), S.end());
  auto it = group_cost.find(S);
  if (it != group_cost.end()) return it->second;
  if (prof) {
    int64_t c = prof->measure_group(*this, S);
    group_cost[S] = c;
    return c;
  }
  if (gm_num > 0) {
    int64_t mx = 0, sum = 0;
    for (int v : S) { mx = std::max(mx, op_cost(v)); sum += op_cost(v); }
    return std::max(mx, (sum * gm_num) / gm_den);
  }
  fail(HIOS_E_STATE, "t(S) unknown for a candidate group (profile, set_group_cost or set_group_model)");
}

std::vector<int64_t> priorities(const Graph& g) {
  std::vector<int64_t> p(g.n, 0);
  for (int k = g.n - 1; k >= 0; --k) {
    int v = g.topo[k];
    int64_t best = 0;
    for (int e : g.ops[v].out_edges) best = std::max(best, g.edge_cost(e) + p[g.edges[e].dst]);
    p[v] = g.op_cost(v) + best;
  }
  return p;
}

std::vector<int> priority_order(const Graph& g) {
  auto p = priorities(g);
  std::vector<int> order(g.n);
  for (int i = 0; i < g.n; ++i) order[i] = i;
  std::sort(order.begin(), order.end(), [&](int a, int b) {
    if (p[a] != p[b]) return p[a] > p[b];
    return g.topo_pos[a] < g.topo_pos[b];
  });
  return order;
}

// ------------------------------------------------ longest valid path (C3, C4)
static std::vector<int> longest_valid_path(const Graph& g, const std::vector<char>& unsched,
                                           const std::vector<int>& rank) {
  const int n = g.n;
  std::vector<int64_t> start(n, 0), end(n, 0);
  std::vector<char> clean(n, 1);
  // unique successor lists inside G' with max parallel-edge weight
  std::vector<std::vector<std::pair<int, int64_t>>> succ(n);
  for (int e = 0; e < (int)g.edges.size(); ++e) {
    int u = g.edges[e].src, v = g.edges[e].dst;
    int64_t c = g.edge_cost(e);
    if (unsched[u] && unsched[v]) {
      bool found = false;
      for (auto& sc : succ[u]) if (sc.first == v) { sc.second = std::max(sc.second, c); found = true; }
      if (!found) succ[u].push_back({v, c});
    } else if (!unsched[u] && unsched[v]) {
      start[v] = std::max(start[v], c); clean[v] = 0;
    } else if (unsched[u] && !unsched[v]) {
      end[u] = std::max(end[u], c); clean[u] = 0;
    }
  }
  // tail(v): best path starting at v with v not the first vertex.  Among equal
  // lengths the lexicographically smallest rank sequence wins; since every
  // candidate starts with v, stopping ([v]) beats continuing ([v, u, ...]),
  // and between continuations the smaller rank(u) wins.
  std::vector<int64_t> tl(n, 0);
  std::vector<int> tn(n, -1);
  for (int k = n - 1; k >= 0; --k) {
    int v = g.topo[k];
    if (!unsched[v]) continue;
    int64_t bl = g.op_cost(v) + end[v];
    int bn = -1;
    if (clean[v]) {
      for (auto& sc : succ[v]) {
        int64_t c = g.op_cost(v) + sc.second + tl[sc.first];
        if (c > bl || (c == bl && bn >= 0 && rank[sc.first] < rank[bn])) { bl = c; bn = sc.first; }
      }
    }
    tl[v] = bl;
    tn[v] = bn;
  }
  int64_t best_len = std::numeric_limits<int64_t>::min();
  int best_v = -1, best_next = -1;
  for (int v = 0; v < n; ++v) {
    if (!unsched[v]) continue;
    int64_t bl = start[v] + g.op_cost(v) + end[v];
    int bn = -1;
    for (auto& sc : succ[v]) {
      int64_t c = start[v] + g.op_cost(v) + sc.second + tl[sc.first];
      if (c > bl || (c == bl && bn >= 0 && rank[sc.first] < rank[bn])) { bl = c; bn = sc.first; }
    }
    if (bl > best_len || (bl == best_len && rank[v] < rank[best_v])) {
      best_len = bl; best_v = v; best_next = bn;
    }
  }
  std::vector<int> P{best_v};
  for (int u = best_next; u >= 0; u = tn[u]) P.push_back(u);
  return P;
}

// ------------------------------------ list scheduling (Alg. 1 L10-13, C1, C5)
static int64_t list_schedule(const Graph& g, const std::vector<int>& gpu, const std::vector<int>& order,
                             int M, std::vector<std::vector<int>>* seq) {
  std::vector<int64_t> ready(M, 0), F(g.n, 0);
  int64_t L = 0;
  if (seq) seq->assign(M, {});
  for (int v : order) {
    int gv = gpu[v];
    if (gv < 0) continue;
    int64_t st = ready[gv];
    for (int e : g.ops[v].in_edges) {
      int u = g.edges[e].src;
      if (gpu[u] < 0) continue;
      st = std::max(st, F[u] + (gpu[u] != gv ? g.edge_cost(e) : 0));
    }
    F[v] = st + g.op_cost(v);
    ready[gv] = F[v];
    L = std::max(L, F[v]);
    if (seq) (*seq)[gv].push_back(v);
  }
  return L;
}

// ------------------------------------------------ cost-model simulator (§III)
SimResult simulate(Graph& g, const std::vector<std::vector<std::vector<int>>>& Q) {
  SimResult r{false, 0, {}, {}};
  const int M = (int)Q.size();
  std::vector<int> base(M + 1, 0);
  for (int i = 0; i < M; ++i) base[i + 1] = base[i] + (int)Q[i].size();
  const int NS = base[M];
  std::vector<int> sid(g.n, -1), sgpu(NS);
  for (int i = 0; i < M; ++i)
    for (int j = 0; j < (int)Q[i].size(); ++j) {
      sgpu[base[i] + j] = i;
      for (int v : Q[i][j]) sid[v] = base[i] + j;
    }
  std::vector<std::vector<std::pair<int, int64_t>>> succ(NS);
  std::vector<int> indeg(NS, 0);
  for (int i = 0; i < M; ++i)
    for (int j = 1; j < (int)Q[i].size(); ++j) {
      succ[base[i] + j - 1].push_back({base[i] + j, 0});
      indeg[base[i] + j]++;
    }
  for (int e = 0; e < (int)g.edges.size(); ++e) {
    int su = sid[g.edges[e].src], sv = sid[g.edges[e].dst];
    if (su < 0 || sv < 0) continue;
    if (su == sv) return r;  // dependent ops in one stage
    succ[su].push_back({sv, sgpu[su] != sgpu[sv] ? g.edge_cost(e) : 0});
    indeg[sv]++;
  }
  std::vector<int64_t> start(NS, 0), finish(NS, 0);
  std::vector<int> stack;
  for (int s = 0; s < NS; ++s) if (!indeg[s]) stack.push_back(s);
  int done = 0;
  while (!stack.empty()) {
    int s = stack.back(); stack.pop_back();
    int i = sgpu[s];
    finish[s] = start[s] + g.stage_cost(Q[i][s - base[i]]);
    r.L = std::max(r.L, finish[s]);
    ++done;
    for (auto& x : succ[s]) {
      start[x.first] = std::max(start[x.first], finish[s] + x.second);
      if (--indeg[x.first] == 0) stack.push_back(x.first);
    }
  }
  if (done != NS) return r;  // cycle: deadlock
  r.ok = true;
  r.start.resize(M); r.finish.resize(M);
  for (int i = 0; i < M; ++i) {
    r.start[i].assign(start.begin() + base[i], start.begin() + base[i + 1]);
    r.finish[i].assign(finish.begin() + base[i], finish.begin() + base[i + 1]);
  }
  return r;
}

// ------------------------------------------------------ Alg. 2 (C7 - C11)
static void parallelize(Graph& g, Schedule& s, const std::vector<int>& order) {
  auto& Q = s.Q;
  auto r0 = simulate(g, Q);
  if (!r0.ok) fail(HIOS_E_CYCLE, "inter-GPU schedule deadlocks");
  int64_t L = r0.L;
  for (int i = 0; i + 1 < g.n; ++i) {
    int v = order[i];
    int gi = -1, j = -1;
    for (int a = 0; a < (int)Q.size() && gi < 0; ++a)
      for (int b = 0; b < (int)Q[a].size(); ++b)
        if (std::find(Q[a][b].begin(), Q[a][b].end(), v) != Q[a][b].end()) { gi = a; j = b; break; }
    if (Q[gi][j].size() > 1) continue;  // C10: already grouped
    int64_t best_L = L;
    std::vector<std::vector<std::vector<int>>> best_Q;
    bool have = false;
    std::vector<int> W{v};
    for (int p = 1; p < s.w; ++p) {
      if (j + p >= (int)Q[gi].size() || Q[gi][j + p].size() > 1) break;
      int u = Q[gi][j + p][0];
      bool ind = true;
      for (int x : W) ind = ind && g.independent(u, x);
      if (!ind) break;  // C8: stop growing at the first dependent pair
      W.push_back(u);
      auto Q2 = Q;
      std::vector<std::vector<int>> row(Q2[gi].begin(), Q2[gi].begin() + j);
      row.push_back(W);
      row.insert(row.end(), Q2[gi].begin() + j + p + 1, Q2[gi].end());
      Q2[gi] = std::move(row);
      auto r2 = simulate(g, Q2);
      if (!r2.ok) continue;  // C11: merging creates a cycle
      if (r2.L < best_L) { best_L = r2.L; best_Q = std::move(Q2); have = true; }
    }
    if (have) { Q = std::move(best_Q); L = best_L; }  // C9: commit only if L' < L
  }
  s.L = L;
}

// ------------------------------------------------------------ Alg. 1
void hios_lp(Graph& g, int M, int w, Schedule& s) {
  s.M = M;
  s.w = w;
  auto order = priority_order(g);
  std::vector<int> rank(g.n);
  for (int i = 0; i < g.n; ++i) rank[order[i]] = i;
  std::vector<char> unsched(g.n, 1);
  int left = g.n;
  std::vector<int> gpu(g.n, -1);
  while (left > 0) {
    auto P = longest_valid_path(g, unsched, rank);
    for (int v : P) { unsched[v] = 0; --left; }
    int64_t best_L = std::numeric_limits<int64_t>::max();
    int best_i = 0;
    for (int i = 0; i < M; ++i) {
      for (int v : P) gpu[v] = i;
      int64_t L2 = list_schedule(g, gpu, order, M, nullptr);
      if (L2 < best_L) { best_L = L2; best_i = i; }  // Alg. 1 L14: first index wins ties
    }
    for (int v : P) gpu[v] = best_i;
  }
  std::vector<std::vector<int>> seq;
  list_schedule(g, gpu, order, M, &seq);
  s.Q.assign(M, {});
  for (int i = 0; i < M; ++i)
    for (int v : seq[i]) s.Q[i].push_back({v});
  parallelize(g, s, order);  // Alg. 1 L17
}

// ------------------------------------------------------------ Alg. 3
// HIOS-MR (garbled pseudo-code reconstructed per C17):
// n x M table of (earliest finish t_{i,j} of v_i on GPU j, GPU g_{i,j} of
// v_{i-1} in that recorded schedule), then back-track and Alg. 2.
void hios_mr(Graph& g, int M, int w, Schedule& s) {
  s.M = M;
  s.w = w;
  auto order = priority_order(g);
  const int n = g.n;
  std::vector<int> pos(n);
  for (int i = 0; i < n; ++i) pos[order[i]] = i;
  const int64_t INF = std::numeric_limits<int64_t>::max();
  std::vector<int64_t> T((size_t)n * M, INF);
  std::vector<int> Gb((size_t)n * M, 0);
  T[0] = g.op_cost(order[0]);  // v_1 on GPU 1 (L5)
  std::vector<int64_t> tF(n, 0);
  std::vector<int> gp(n, -1);
  std::vector<int64_t> ready(M, 0);
  for (int i = 1; i < n; ++i) {
    const int vi = order[i];
    const int kmax = std::min(M, i);
    for (int k = 0; k < kmax; ++k) {
      if (T[(size_t)(i - 1) * M + k] == INF) continue;
      // recorded schedule of v_1..v_{i-1} with v_{i-1} on GPU k (L9-12)
      int m = k;
      std::fill(ready.begin(), ready.end(), 0);
      for (int l = i - 1; l >= 0; --l) {
        const int vl = order[l];
        tF[vl] = T[(size_t)l * M + m];
        gp[vl] = m;
        ready[m] = std::max(ready[m], tF[vl]);
        m = Gb[(size_t)l * M + m];
      }
      const int jmax = std::min(M, i + 1);
      for (int j = 0; j < jmax; ++j) {
        int64_t tk = ready[j];  // L14
        for (int e : g.ops[vi].in_edges) {  // L15-19
          const int u = g.edges[e].src;
          if (pos[u] >= i) continue;
          tk = std::max(tk, gp[u] == j ? tF[u] : tF[u] + g.edge_cost(e));
        }
        const int64_t f = tk + g.op_cost(vi);
        if (T[(size_t)i * M + j] > f) {  // L20-21 (first k wins ties)
          T[(size_t)i * M + j] = f;
          Gb[(size_t)i * M + j] = k;
        }
      }
    }
  }
  int J = 0;  // L22
  for (int j = 1; j < M; ++j)
    if (T[(size_t)(n - 1) * M + j] < T[(size_t)(n - 1) * M + J]) J = j;
  std::vector<int> gpu(n, 0);
  int m = J;
  for (int i = n - 1; i >= 0; --i) {  // L24-25
    gpu[order[i]] = m;
    m = Gb[(size_t)i * M + m];
  }
  s.Q.assign(M, {});
  for (int v : order) s.Q[gpu[v]].push_back({v});
  parallelize(g, s, order);  // L27
}

// ------------------------------------------------ IOS (exact, one GPU)
// The paper's single-GPU comparator ("an exact
// algorithm for the optimal schedule in a single GPU", dynamic programming):
// the stage sequence (stages = <= w pairwise-independent ready ops) that
// minimises L = sum t(S).  DP over the finished set D:
//   f(V) = 0,  f(D) = min_E t(E) + f(D | E).
// Exact decomposition at cut vertices (ops comparable with every other op:
// such an op is always a stage of its own and splits G into independent
// sub-problems), then a memoised DP per block (bitmasks).  Blocks of more
// than 32 ops are cut into topological-order chunks (exact per chunk).
// Enumeration: ready ops ascending, subsets in combinations order, sizes
// ascending, first strict minimum -- as oracle/sched.py: ios_dp.
void hios_ios(Graph& g, int w, Schedule& s, int64_t max_states) {
  s.M = 1;
  s.w = w;
  const int n = g.n;
  // cut vertices
  std::vector<int> before(n, 0), after(n, 0);
  for (int u = 0; u < n; ++u)
    for (int v = 0; v < n; ++v)
      if (g.reaches(u, v)) { ++after[u]; ++before[v]; }
  std::vector<char> cut(n, 0);
  for (int v = 0; v < n; ++v) cut[v] = before[v] + after[v] == n - 1;
  // block of a non-cut op = number of cut vertices before it
  std::vector<int> cuts;
  for (int v : g.topo) if (cut[v]) cuts.push_back(v);
  std::vector<std::vector<int>> blocks(cuts.size() + 1);
  for (int v : g.topo) {
    if (cut[v]) continue;
    int b = 0;
    for (int c : cuts) b += g.reaches(c, v) ? 1 : 0;
    blocks[b].push_back(v);
  }
  std::vector<std::vector<int>> stages;
  int64_t states = 0;
  auto solve_block = [&](std::vector<int> ops) {
    if (ops.empty()) return;
    std::sort(ops.begin(), ops.end());
    const int m = (int)ops.size();
    std::vector<uint64_t> pred_mask(m, 0), indep(m, 0);
    for (int i = 0; i < m; ++i)
      for (int j = 0; j < m; ++j) {
        if (g.reaches(ops[j], ops[i])) {
          // only direct preds matter for readiness, but any ancestor in the
          // block being finished first is implied by downward closure
          pred_mask[i] |= 1ull << j;
        }
        if (g.independent(ops[i], ops[j])) indep[i] |= 1ull << j;
      }
    const uint64_t full = m == 64 ? ~0ull : ((1ull << m) - 1);
    std::unordered_map<uint64_t, std::pair<int64_t, uint64_t>> memo;
    memo[full] = {0, 0};
    std::function<int64_t(uint64_t)> f = [&](uint64_t D) -> int64_t {
      auto it = memo.find(D);
      if (it != memo.end()) return it->second.first;
      if (++states > max_states) fail(HIOS_E_UNSUPPORTED, "IOS DP: state budget exceeded");
      int ready[64];
      int r = 0;
      for (int i = 0; i < m; ++i)
        if (!((D >> i) & 1) && (pred_mask[i] & ~D) == 0) ready[r++] = i;
      int64_t best = std::numeric_limits<int64_t>::max();
      uint64_t arg = 0;
      int idx[8];
      for (int k = 1; k <= std::min(w, r); ++k) {
        for (int q = 0; q < k; ++q) idx[q] = q;
        while (true) {
          bool ok = true;
          uint64_t E = 0;
          for (int q = 0; q < k && ok; ++q) {
            const int a = ready[idx[q]];
            for (int q2 = 0; q2 < q; ++q2)
              if (!((indep[a] >> ready[idx[q2]]) & 1)) { ok = false; break; }
            E |= 1ull << a;
          }
          if (ok) {
            std::vector<int> S;
            for (int q = 0; q < k; ++q) S.push_back(ops[ready[idx[q]]]);
            const int64_t c = g.stage_cost(S) + f(D | E);
            if (c < best) { best = c; arg = E; }
          }
          // next combination (lexicographic)
          int q = k - 1;
          while (q >= 0 && idx[q] == r - k + q) --q;
          if (q < 0) break;
          ++idx[q];
          for (int q2 = q + 1; q2 < k; ++q2) idx[q2] = idx[q2 - 1] + 1;
        }
      }
      memo[D] = {best, arg};
      return best;
    };
    f(0);
    uint64_t D = 0;
    while (D != full) {
      const uint64_t E = memo[D].second;
      std::vector<int> S;
      for (int i = 0; i < m; ++i)
        if ((E >> i) & 1) S.push_back(ops[i]);
      stages.push_back(S);
      D |= E;
    }
  };
  // blocks of more than `chunk` ops (no cut vertex inside, e.g. NASNet's
  // two-input cells) are cut into consecutive topological-order chunks, as
  // IOS itself partitions large graphs; the DP is then exact per chunk
  const int chunk = 32;
  auto solve = [&](const std::vector<int>& ops) {  // ops in topological order
    for (size_t i = 0; i < ops.size(); i += chunk)
      solve_block(std::vector<int>(ops.begin() + i, ops.begin() + std::min(ops.size(), i + chunk)));
  };
  solve(blocks[0]);
  for (size_t c = 0; c < cuts.size(); ++c) {
    stages.push_back({cuts[c]});
    solve(blocks[c + 1]);
  }
  s.Q.assign(1, stages);
}

void finalize_schedule(Schedule& s) {
  Graph& g = *s.g;
  s.gpu_of.assign(g.n, -1);
  s.stage_of.assign(g.n, -1);
  for (int i = 0; i < (int)s.Q.size(); ++i)
    for (int j = 0; j < (int)s.Q[i].size(); ++j) {
      auto& S = s.Q[i][j];
      if (S.empty() || (int)S.size() > std::max(s.w, 1))
        fail(HIOS_E_INVALID, "stage size out of [1, w]");
      for (size_t a = 0; a < S.size(); ++a) {
        int v = S[a];
        if (v < 0 || v >= g.n) fail(HIOS_E_INVALID, "op id out of range");
        if (s.gpu_of[v] >= 0) fail(HIOS_E_INVALID, "op " + std::to_string(v) + " scheduled twice");
        s.gpu_of[v] = i;
        s.stage_of[v] = j;
        for (size_t b = a + 1; b < S.size(); ++b)
          if (!g.independent(v, S[b])) fail(HIOS_E_INVALID, "dependent ops in one stage");
      }
    }
  for (int v = 0; v < g.n; ++v)
    if (s.gpu_of[v] < 0) fail(HIOS_E_INVALID, "op " + std::to_string(v) + " unscheduled");
  auto r = simulate(g, s.Q);
  if (!r.ok) fail(HIOS_E_CYCLE, "schedule deadlocks (cycle in the stage graph)");
  s.L = r.L;
}

}  // namespace hios
