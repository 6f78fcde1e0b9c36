// graph.cpp -- the computation graph G = (V, E) of PAPER.md §III-A:
// validation, Kahn topological order, shape inference and the reachability
// bitsets used by Alg. 2's independence test.
#include <algorithm>
#include <queue>

#include "internal.h"

namespace hios {

int out_size(int h, int k, int s, int p, int d, int ceil_mode) {
  int num = h + 2 * p - d * (k - 1) - 1;
  if (num < 0) return 0;
  int o;
  if (ceil_mode) {
    o = (num + s - 1) / s + 1;
    if ((o - 1) * s >= h + p) o -= 1;
  } else {
    o = num / s + 1;
  }
  return o;
}

static void need(bool c, hios_status code, const std::string& m) {
  if (!c) fail(code, m);
}

std::shared_ptr<Graph> build_graph(const hios_op* ops, int n_ops, const hios_edge* edges, int n_edges,
                                   int in_c, int in_h, int in_w, hios_dtype dtype) {
  need(ops && n_ops > 0, HIOS_E_INVALID, "no ops");
  need(n_edges >= 0 && (n_edges == 0 || edges), HIOS_E_INVALID, "bad edges");
  need(in_c > 0 && in_h > 0 && in_w > 0, HIOS_E_INVALID, "bad input shape");
  need(dtype == HIOS_F32 || dtype == HIOS_BF16, HIOS_E_INVALID, "bad dtype");
  auto G = std::make_shared<Graph>();
  Graph& g = *G;
  g.n = n_ops;
  g.in_c = in_c;
  g.in_h = in_h;
  g.in_w = in_w;
  g.dtype = dtype;
  g.ops.resize(n_ops);
  for (int i = 0; i < n_ops; ++i) {
    const hios_op& a = ops[i];
    Op& o = g.ops[i];
    need(a.kind >= HIOS_OP_INPUT && a.kind <= HIOS_OP_IDENTITY, HIOS_E_INVALID,
         "op " + std::to_string(i) + ": bad kind");
    o.kind = a.kind;
    o.in_c = a.in_c; o.out_c = a.out_c;
    o.kh = a.kh; o.kw = a.kw; o.sh = a.sh; o.sw = a.sw; o.ph = a.ph; o.pw = a.pw;
    o.dh = a.dh > 0 ? a.dh : 1; o.dw = a.dw > 0 ? a.dw : 1;
    o.relu = a.relu; o.pre_relu = a.pre_relu; o.ceil_mode = a.ceil_mode;
    o.cip = a.count_include_pad; o.reps = a.reps > 0 ? a.reps : 1;
    o.cost = a.cost_ns;
    bool spatial = o.kind == HIOS_OP_CONV || o.kind == HIOS_OP_SEPCONV ||
                   o.kind == HIOS_OP_MAXPOOL || o.kind == HIOS_OP_AVGPOOL;
    if (spatial) {
      need(o.kh >= 1 && o.kw >= 1 && o.sh >= 1 && o.sw >= 1 && o.ph >= 0 && o.pw >= 0,
           HIOS_E_INVALID, "op " + std::to_string(i) + ": bad window");
      need(o.kh <= 15 && o.kw <= 15, HIOS_E_UNSUPPORTED, "kernel larger than 15");
    }
    if (o.kind == HIOS_OP_SEPCONV) need(o.dh == 1 && o.dw == 1, HIOS_E_UNSUPPORTED, "dilated sepconv");
    if (o.kind == HIOS_OP_MAXPOOL || o.kind == HIOS_OP_AVGPOOL)
      need(o.ph * 2 <= o.kh && o.pw * 2 <= o.kw, HIOS_E_INVALID, "pool pad > kernel/2");
  }
  g.edges.resize(n_edges);
  for (int e = 0; e < n_edges; ++e) {
    const hios_edge& a = edges[e];
    need(a.src >= 0 && a.src < n_ops && a.dst >= 0 && a.dst < n_ops, HIOS_E_INVALID,
         "edge " + std::to_string(e) + ": endpoint out of range");
    need(a.src != a.dst, HIOS_E_INVALID, "edge " + std::to_string(e) + ": self loop");
    g.edges[e] = Edge{a.src, a.dst, a.slot, a.cost_ns};
    g.ops[a.src].out_edges.push_back(e);
    g.ops[a.dst].in_edges.push_back(e);
  }
  for (int i = 0; i < n_ops; ++i) {
    Op& o = g.ops[i];
    std::sort(o.in_edges.begin(), o.in_edges.end(),
              [&](int a, int b) { return g.edges[a].slot < g.edges[b].slot; });
    for (size_t k = 0; k < o.in_edges.size(); ++k)
      need(g.edges[o.in_edges[k]].slot == (int)k, HIOS_E_INVALID,
           "op " + std::to_string(i) + ": input slots must be 0..n_in-1");
    int nin = (int)o.in_edges.size();
    switch (o.kind) {
      case HIOS_OP_INPUT:
        need(nin == 0, HIOS_E_INVALID, "input op has inputs");
        need(g.input_op < 0, HIOS_E_INVALID, "more than one input op");
        g.input_op = i;
        break;
      case HIOS_OP_CONV: case HIOS_OP_MAXPOOL: case HIOS_OP_AVGPOOL: case HIOS_OP_GAP:
      case HIOS_OP_LINEAR: case HIOS_OP_IDENTITY:
        need(nin == 1, HIOS_E_INVALID, "op " + std::to_string(i) + " needs exactly one input");
        break;
      default:
        need(nin >= 1, HIOS_E_INVALID, "op " + std::to_string(i) + " has no inputs");
    }
  }
  need(g.input_op >= 0, HIOS_E_INVALID, "graph has no input op");
  // Kahn topological order, smallest id first (shared tie rule with the oracle)
  {
    std::vector<int> indeg(n_ops, 0);
    for (auto& e : g.edges) indeg[e.dst]++;
    std::priority_queue<int, std::vector<int>, std::greater<int>> h;
    for (int i = 0; i < n_ops; ++i) if (!indeg[i]) h.push(i);
    g.topo_pos.assign(n_ops, -1);
    while (!h.empty()) {
      int v = h.top(); h.pop();
      g.topo_pos[v] = (int)g.topo.size();
      g.topo.push_back(v);
      for (int e : g.ops[v].out_edges) if (--indeg[g.edges[e].dst] == 0) h.push(g.edges[e].dst);
    }
    need((int)g.topo.size() == n_ops, HIOS_E_CYCLE, "graph has a cycle");
  }
  // sink
  for (int i = 0; i < n_ops; ++i)
    if (g.ops[i].out_edges.empty()) {
      need(g.sink_op < 0, HIOS_E_INVALID, "graph must have exactly one sink (output) op");
      g.sink_op = i;
    }
  // weights + shapes in topological order
  for (int v : g.topo) {
    Op& o = g.ops[v];
    const hios_op& a = ops[v];
    std::string id = "op " + std::to_string(v);
    auto in = [&](int k) -> Op& { return g.ops[g.edges[o.in_edges[k]].src]; };
    int nin = (int)o.in_edges.size();
    switch (o.kind) {
      case HIOS_OP_INPUT:
        if (o.out_c == 0) o.out_c = in_c;
        need(o.out_c == in_c, HIOS_E_SHAPE, id + ": input channels != in_c");
        o.C = in_c; o.H = in_h; o.W = in_w;
        break;
      case HIOS_OP_CONV: {
        Op& x = in(0);
        if (o.in_c == 0) o.in_c = x.C;
        need(o.in_c == x.C, HIOS_E_SHAPE, id + ": in_c != input channels");
        need(o.out_c > 0, HIOS_E_INVALID, id + ": out_c");
        o.C = o.out_c;
        o.H = out_size(x.H, o.kh, o.sh, o.ph, o.dh, 0);
        o.W = out_size(x.W, o.kw, o.sw, o.pw, o.dw, 0);
        need(a.weight != nullptr, HIOS_E_INVALID, id + ": conv weight is NULL");
        size_t nw = (size_t)o.out_c * o.in_c * o.kh * o.kw;
        o.weight.assign(a.weight, a.weight + nw);
        o.scale.assign(o.out_c, 1.f);
        o.shift.assign(o.out_c, 0.f);
        if (a.scale) o.scale.assign(a.scale, a.scale + o.out_c);
        if (a.shift) o.shift.assign(a.shift, a.shift + o.out_c);
        break;
      }
      case HIOS_OP_SEPCONV: {
        Op& x = in(0);
        for (int k = 1; k < nin; ++k)
          need(in(k).C == x.C && in(k).H == x.H && in(k).W == x.W, HIOS_E_SHAPE, id + ": input shapes differ");
        if (o.in_c == 0) o.in_c = x.C;
        need(o.in_c == x.C, HIOS_E_SHAPE, id + ": in_c != input channels");
        need(o.out_c > 0, HIOS_E_INVALID, id + ": out_c");
        o.C = o.out_c;
        o.H = out_size(x.H, o.kh, o.sh, o.ph, 1, 0);
        o.W = out_size(x.W, o.kw, o.sw, o.pw, 1, 0);
        if (o.reps > 1) {  // later repetitions are stride 1 'same' convs
          need(out_size(o.H, o.kh, 1, o.ph, 1, 0) == o.H && out_size(o.W, o.kw, 1, o.pw, 1, 0) == o.W,
               HIOS_E_SHAPE, id + ": repetitions must preserve the spatial size");
        }
        need(a.weight != nullptr, HIOS_E_INVALID, id + ": sepconv weight is NULL");
        size_t nw = 0;
        for (int r = 0; r < o.reps; ++r) {
          int c = r == 0 ? o.in_c : o.out_c;
          nw += (size_t)c * o.kh * o.kw + (size_t)o.out_c * c;
        }
        o.weight.assign(a.weight, a.weight + nw);
        o.scale.assign((size_t)o.reps * o.out_c, 1.f);
        o.shift.assign((size_t)o.reps * o.out_c, 0.f);
        if (a.scale) o.scale.assign(a.scale, a.scale + (size_t)o.reps * o.out_c);
        if (a.shift) o.shift.assign(a.shift, a.shift + (size_t)o.reps * o.out_c);
        if (a.agg) o.agg.assign(a.agg, a.agg + nin);
        else need(nin == 1, HIOS_E_INVALID, id + ": several inputs need agg weights");
        break;
      }
      case HIOS_OP_MAXPOOL: case HIOS_OP_AVGPOOL: {
        Op& x = in(0);
        o.C = x.C;
        o.H = out_size(x.H, o.kh, o.sh, o.ph, 1, o.ceil_mode);
        o.W = out_size(x.W, o.kw, o.sw, o.pw, 1, o.ceil_mode);
        if (o.out_c == 0) o.out_c = o.C;
        break;
      }
      case HIOS_OP_GAP: {
        Op& x = in(0);
        o.C = x.C; o.H = 1; o.W = 1;
        if (o.out_c == 0) o.out_c = o.C;
        break;
      }
      case HIOS_OP_CONCAT: {
        Op& x = in(0);
        int c = 0;
        for (int k = 0; k < nin; ++k) {
          need(in(k).H == x.H && in(k).W == x.W, HIOS_E_SHAPE, id + ": concat spatial sizes differ");
          c += in(k).C;
        }
        o.C = c; o.H = x.H; o.W = x.W;
        if (o.out_c == 0) o.out_c = c;
        need(o.out_c == c, HIOS_E_SHAPE, id + ": concat out_c");
        break;
      }
      case HIOS_OP_ADD: {
        Op& x = in(0);
        for (int k = 1; k < nin; ++k)
          need(in(k).C == x.C && in(k).H == x.H && in(k).W == x.W, HIOS_E_SHAPE, id + ": add shapes differ");
        o.C = x.C; o.H = x.H; o.W = x.W;
        if (o.out_c == 0) o.out_c = o.C;
        o.agg.assign(nin, 1.f);
        if (a.agg) o.agg.assign(a.agg, a.agg + nin);
        break;
      }
      case HIOS_OP_LINEAR: {
        Op& x = in(0);
        int cin = x.C * x.H * x.W;
        if (o.in_c == 0) o.in_c = cin;
        need(o.in_c == cin, HIOS_E_SHAPE, id + ": linear in_c != flattened input");
        need(o.out_c > 0 && a.weight != nullptr, HIOS_E_INVALID, id + ": linear weight");
        o.C = o.out_c; o.H = 1; o.W = 1;
        o.weight.assign(a.weight, a.weight + (size_t)o.out_c * o.in_c);
        o.shift.assign(o.out_c, 0.f);
        if (a.shift) o.shift.assign(a.shift, a.shift + o.out_c);
        break;
      }
      case HIOS_OP_IDENTITY: {
        Op& x = in(0);
        o.C = x.C; o.H = x.H; o.W = x.W;
        if (o.out_c == 0) o.out_c = o.C;
        break;
      }
    }
    need(o.C > 0 && o.H > 0 && o.W > 0, HIOS_E_SHAPE, id + ": empty output");
  }
  // reachability bitsets (reverse topological order)
  g.words = (n_ops + 63) / 64;
  g.reach.assign((size_t)n_ops * g.words, 0ull);
  for (int k = n_ops - 1; k >= 0; --k) {
    int u = g.topo[k];
    uint64_t* ru = &g.reach[(size_t)u * g.words];
    for (int e : g.ops[u].out_edges) {
      int v = g.edges[e].dst;
      ru[v >> 6] |= 1ull << (v & 63);
      const uint64_t* rv = &g.reach[(size_t)v * g.words];
      for (int w = 0; w < g.words; ++w) ru[w] |= rv[w];
    }
  }
  return G;
}

}  // namespace hios
