// internal.h -- shared host-side structures of the HIOS executor (not ABI).
#pragma once
#include <cstdint>
#include <map>
#include <memory>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/hios.h"

namespace hios {

struct Error : std::runtime_error {
  hios_status code;
  Error(hios_status c, const std::string& m) : std::runtime_error(m), code(c) {}
};
[[noreturn]] inline void fail(hios_status c, const std::string& m) { throw Error(c, m); }

struct Op {
  int kind = 0;
  int in_c = 0, out_c = 0, kh = 1, kw = 1, sh = 1, sw = 1, ph = 0, pw = 0, dh = 1, dw = 1;
  int relu = 0, pre_relu = 0, ceil_mode = 0, cip = 1, reps = 1;
  std::vector<float> weight, scale, shift, agg;
  int64_t cost = -1;
  // inferred output shape
  int C = 0, H = 0, W = 0;
  // incident edges: in_edges sorted by slot
  std::vector<int> in_edges, out_edges;
};

struct Edge {
  int src = 0, dst = 0, slot = 0;
  int64_t cost = -1;
};

struct Graph;
// exec side: device measurement of t(S) for a candidate group
class Profiler {
 public:
  virtual ~Profiler() {}
  virtual int64_t measure_group(Graph& g, const std::vector<int>& S) = 0;
};

struct Graph {
  int n = 0;
  std::vector<Op> ops;
  std::vector<Edge> edges;
  int in_c = 0, in_h = 0, in_w = 0;
  hios_dtype dtype = HIOS_BF16;
  int input_op = -1, sink_op = -1;
  std::vector<int> topo_pos;   // Kahn order, smallest id first
  std::vector<int> topo;       // ops in that order
  int words = 0;               // reachability bitset words per op
  std::vector<uint64_t> reach; // reach[u*words + v/64] bit = path u ->+ v
  std::map<std::vector<int>, int64_t> group_cost;  // sorted op set -> t(S)
  int gm_num = 0, gm_den = 1;
  std::shared_ptr<Profiler> prof;

  bool reaches(int u, int v) const { return (reach[(size_t)u * words + (v >> 6)] >> (v & 63)) & 1ull; }
  bool independent(int a, int b) const { return a != b && !reaches(a, b) && !reaches(b, a); }
  int64_t op_cost(int v) const {
    if (ops[v].cost < 0) fail(HIOS_E_STATE, "t(v) unknown for op " + std::to_string(v) + " (profile or inject costs)");
    return ops[v].cost;
  }
  int64_t edge_cost(int e) const {
    if (edges[e].cost < 0) fail(HIOS_E_STATE, "t(u,v) unknown for edge " + std::to_string(e));
    return edges[e].cost;
  }
  int64_t stage_cost(const std::vector<int>& S);  // t(S) (singletons: t(v))
};

struct Executor;  // exec.cu

struct Schedule {
  std::shared_ptr<Graph> g;
  int M = 1, w = 1;
  std::vector<std::vector<std::vector<int>>> Q;  // Q[gpu][stage] = ops
  int64_t L = 0;
  std::vector<int> gpu_of, stage_of;
  // placement
  std::vector<int> devices;  // per logical GPU
  std::vector<int> owner;    // per logical GPU: process rank (empty = all local)
  int rank = 0;
  int transport = HIOS_TRANSPORT_PEER;
  int stage_mode = HIOS_STAGE_STREAMS;
  std::unique_ptr<Executor> exec;
  ~Schedule();
};

// graph.cpp
std::shared_ptr<Graph> build_graph(const hios_op* ops, int n_ops, const hios_edge* edges, int n_edges,
                                   int in_c, int in_h, int in_w, hios_dtype dtype);
int out_size(int h, int k, int s, int p, int d, int ceil_mode);

// sched.cpp
std::vector<int64_t> priorities(const Graph& g);
std::vector<int> priority_order(const Graph& g);
struct SimResult { bool ok; int64_t L; std::vector<std::vector<int64_t>> start, finish; };
SimResult simulate(Graph& g, const std::vector<std::vector<std::vector<int>>>& Q);
void hios_lp(Graph& g, int M, int w, Schedule& s);
void hios_mr(Graph& g, int M, int w, Schedule& s);
void hios_ios(Graph& g, int w, Schedule& s, int64_t max_states);
void finalize_schedule(Schedule& s);  // gpu_of/stage_of + validation (C6)

}  // namespace hios
