// api.cu -- the extern "C" boundary declared in include/hios.h.  Every entry
// point converts exceptions into a hios_status + thread-local message.
#include <cstring>
#include <string>

#include "exec.h"

struct hios_graph_s {
  std::shared_ptr<hios::Graph> g;
};
struct hios_schedule_s {
  std::unique_ptr<hios::Schedule> s;
};

namespace hios {
Schedule::~Schedule() {}
std::shared_ptr<Profiler> run_profile(std::shared_ptr<Graph> G, const int32_t* devices, int32_t n_devices,
                                      int32_t reps);
}  // namespace hios

static thread_local std::string g_err;

template <typename F>
static hios_status guard(F&& f) {
  try {
    g_err.clear();
    f();
    return HIOS_OK;
  } catch (const hios::Error& e) {
    g_err = e.what();
    return e.code;
  } catch (const std::bad_alloc&) {
    g_err = "out of host memory";
    return HIOS_E_OOM;
  } catch (const std::exception& e) {
    g_err = e.what();
    return HIOS_E_INVALID;
  } catch (...) {
    g_err = "unknown error";
    return HIOS_E_INVALID;
  }
}

#define NEED(c, code, msg) \
  do {                     \
    if (!(c)) hios::fail(code, msg); \
  } while (0)

extern "C" {

const char* hios_last_error(void) { return g_err.c_str(); }
int32_t hios_abi_version(void) { return HIOS_ABI_VERSION; }

hios_status hios_graph_create(const hios_op* ops, int32_t n_ops, const hios_edge* edges, int32_t n_edges,
                              int32_t in_c, int32_t in_h, int32_t in_w, hios_dtype dtype, hios_graph* out) {
  if (out) *out = nullptr;
  return guard([&] {
    NEED(out, HIOS_E_INVALID, "out is NULL");
    auto g = hios::build_graph(ops, n_ops, edges, n_edges, in_c, in_h, in_w, dtype);
    auto* h = new hios_graph_s;
    h->g = g;
    *out = h;
  });
}

void hios_graph_destroy(hios_graph g) { delete g; }

hios_status hios_graph_shape(hios_graph g, int32_t op, int32_t* c, int32_t* h, int32_t* w) {
  return guard([&] {
    NEED(g && op >= 0 && op < g->g->n, HIOS_E_INVALID, "bad graph/op");
    const auto& o = g->g->ops[op];
    if (c) *c = o.C;
    if (h) *h = o.H;
    if (w) *w = o.W;
  });
}

hios_status hios_set_op_cost(hios_graph g, int32_t op, int64_t ns) {
  return guard([&] {
    NEED(g && op >= 0 && op < g->g->n, HIOS_E_INVALID, "bad graph/op");
    g->g->ops[op].cost = ns;
  });
}

hios_status hios_set_edge_cost(hios_graph g, int32_t e, int64_t ns) {
  return guard([&] {
    NEED(g && e >= 0 && e < (int)g->g->edges.size(), HIOS_E_INVALID, "bad graph/edge");
    g->g->edges[e].cost = ns;
  });
}

hios_status hios_set_group_cost(hios_graph g, const int32_t* ops, int32_t n, int64_t ns) {
  return guard([&] {
    NEED(g && ops && n >= 2, HIOS_E_INVALID, "group needs >= 2 ops");
    std::vector<int> S(ops, ops + n);
    for (int v : S) NEED(v >= 0 && v < g->g->n, HIOS_E_INVALID, "op out of range");
    std::sort(S.begin(), S.end());
    g->g->group_cost[S] = ns;
  });
}

hios_status hios_set_group_model(hios_graph g, int32_t num, int32_t den) {
  return guard([&] {
    NEED(g && num >= 0 && den > 0, HIOS_E_INVALID, "bad model");
    g->g->gm_num = num;
    g->g->gm_den = den;
  });
}

hios_status hios_get_costs(hios_graph g, int64_t* op_ns, int64_t* edge_ns) {
  return guard([&] {
    NEED(g, HIOS_E_INVALID, "graph is NULL");
    if (op_ns)
      for (int v = 0; v < g->g->n; ++v) op_ns[v] = g->g->ops[v].cost;
    if (edge_ns)
      for (size_t e = 0; e < g->g->edges.size(); ++e) edge_ns[e] = g->g->edges[e].cost;
  });
}

hios_status hios_group_cost(hios_graph g, const int32_t* ops, int32_t n, int64_t* ns) {
  return guard([&] {
    NEED(g && ops && ns && n >= 1, HIOS_E_INVALID, "bad arguments");
    std::vector<int> S(ops, ops + n);
    for (int v : S) NEED(v >= 0 && v < g->g->n, HIOS_E_INVALID, "op out of range");
    std::sort(S.begin(), S.end());
    NEED(std::adjacent_find(S.begin(), S.end()) == S.end(), HIOS_E_INVALID, "duplicate op");
    *ns = g->g->stage_cost(S);
  });
}

hios_status hios_profile(hios_graph g, const int32_t* devices, int32_t n_devices, int32_t reps) {
  return guard([&] {
    NEED(g, HIOS_E_INVALID, "graph is NULL");
    NEED(n_devices >= 0 && (n_devices == 0 || devices), HIOS_E_INVALID, "bad devices");
    g->g->prof.reset();
    g->g->prof = hios::run_profile(g->g, devices, n_devices, reps);
  });
}

hios_status hios_schedule_lp(hios_graph g, int32_t n_gpus, int32_t window, hios_schedule* out) {
  if (out) *out = nullptr;
  return guard([&] {
    NEED(g && out, HIOS_E_INVALID, "NULL argument");
    NEED(n_gpus >= 1 && n_gpus <= 64, HIOS_E_INVALID, "n_gpus out of [1, 64]");
    NEED(window >= 1 && window <= 8, HIOS_E_INVALID, "window out of [1, 8]");
    std::unique_ptr<hios::Schedule> s(new hios::Schedule);
    s->g = g->g;
    hios::hios_lp(*g->g, n_gpus, window, *s);
    hios::finalize_schedule(*s);
    auto* h = new hios_schedule_s;
    h->s = std::move(s);
    *out = h;
  });
}

hios_status hios_schedule_mr(hios_graph g, int32_t n_gpus, int32_t window, hios_schedule* out) {
  if (out) *out = nullptr;
  return guard([&] {
    NEED(g && out, HIOS_E_INVALID, "NULL argument");
    NEED(n_gpus >= 1 && n_gpus <= 64, HIOS_E_INVALID, "n_gpus out of [1, 64]");
    NEED(window >= 1 && window <= 8, HIOS_E_INVALID, "window out of [1, 8]");
    std::unique_ptr<hios::Schedule> s(new hios::Schedule);
    s->g = g->g;
    hios::hios_mr(*g->g, n_gpus, window, *s);
    hios::finalize_schedule(*s);
    auto* h = new hios_schedule_s;
    h->s = std::move(s);
    *out = h;
  });
}

hios_status hios_schedule_ios(hios_graph g, int32_t window, int64_t max_states, hios_schedule* out) {
  if (out) *out = nullptr;
  return guard([&] {
    NEED(g && out, HIOS_E_INVALID, "NULL argument");
    NEED(window >= 1 && window <= 8, HIOS_E_INVALID, "window out of [1, 8]");
    std::unique_ptr<hios::Schedule> s(new hios::Schedule);
    s->g = g->g;
    hios::hios_ios(*g->g, window, *s, max_states > 0 ? max_states : (int64_t)1 << 22);
    hios::finalize_schedule(*s);
    auto* h = new hios_schedule_s;
    h->s = std::move(s);
    *out = h;
  });
}

hios_status hios_schedule_import(hios_graph g, int32_t n_gpus, int32_t window, const int32_t* op_gpu,
                                 const int32_t* op_stage, hios_schedule* out) {
  if (out) *out = nullptr;
  return guard([&] {
    NEED(g && out && op_gpu && op_stage, HIOS_E_INVALID, "NULL argument");
    NEED(n_gpus >= 1 && window >= 1, HIOS_E_INVALID, "bad n_gpus/window");
    auto& G = *g->g;
    std::unique_ptr<hios::Schedule> s(new hios::Schedule);
    s->g = g->g;
    s->M = n_gpus;
    s->w = window;
    s->Q.assign(n_gpus, {});
    for (int v = 0; v < G.n; ++v) {
      NEED(op_gpu[v] >= 0 && op_gpu[v] < n_gpus, HIOS_E_INVALID, "op_gpu out of range");
      NEED(op_stage[v] >= 0 && op_stage[v] < G.n, HIOS_E_INVALID, "op_stage out of range");
      auto& q = s->Q[op_gpu[v]];
      if ((int)q.size() <= op_stage[v]) q.resize(op_stage[v] + 1);
      q[op_stage[v]].push_back(v);
    }
    for (auto& q : s->Q)
      for (auto& S : q) NEED(!S.empty(), HIOS_E_INVALID, "empty stage index");
    hios::finalize_schedule(*s);
    auto* h = new hios_schedule_s;
    h->s = std::move(s);
    *out = h;
  });
}

void hios_schedule_destroy(hios_schedule s) {
  if (!s) return;
  try {
    delete s;
  } catch (...) {
  }
}

hios_status hios_schedule_latency_ns(hios_schedule s, int64_t* predicted) {
  return guard([&] {
    NEED(s && predicted, HIOS_E_INVALID, "NULL argument");
    *predicted = s->s->L;
  });
}

hios_status hios_schedule_stages(hios_schedule s, int32_t* op_gpu, int32_t* op_stage, int32_t* n_stages) {
  return guard([&] {
    NEED(s, HIOS_E_INVALID, "NULL schedule");
    auto& S = *s->s;
    for (int v = 0; v < S.g->n; ++v) {
      if (op_gpu) op_gpu[v] = S.gpu_of[v];
      if (op_stage) op_stage[v] = S.stage_of[v];
    }
    if (n_stages)
      for (int i = 0; i < S.M; ++i) n_stages[i] = (int)S.Q[i].size();
  });
}

hios_status hios_schedule_place(hios_schedule s, const int32_t* devices, int32_t n) {
  return guard([&] {
    NEED(s && devices && n == s->s->M, HIOS_E_INVALID, "need one device per logical GPU");
    NEED(!s->s->exec, HIOS_E_STATE, "placement after the first run");
    s->s->devices.assign(devices, devices + n);
  });
}

hios_status hios_schedule_bind_rank(hios_schedule s, const int32_t* owner, int32_t n, int32_t rank) {
  return guard([&] {
    NEED(s && owner && n == s->s->M, HIOS_E_INVALID, "need one owner per logical GPU");
    NEED(!s->s->exec, HIOS_E_STATE, "bind after the first run");
    s->s->owner.assign(owner, owner + n);
    s->s->rank = rank;
  });
}

static hios::Executor& ensure_exec(hios::Schedule& S) {
  if (!S.exec) S.exec.reset(new hios::Executor(S));
  return *S.exec;
}

hios_status hios_schedule_transport(hios_schedule s, int32_t transport) {
  return guard([&] {
    NEED(s, HIOS_E_INVALID, "NULL schedule");
    NEED(transport == HIOS_TRANSPORT_PEER || transport == HIOS_TRANSPORT_COPY || transport == HIOS_TRANSPORT_NCCL,
         HIOS_E_INVALID, "unknown transport");
    NEED(!s->s->exec, HIOS_E_STATE, "set the transport before the first run / IPC export");
    s->s->transport = transport;
  });
}

hios_status hios_schedule_stage_mode(hios_schedule s, int32_t mode) {
  return guard([&] {
    NEED(s, HIOS_E_INVALID, "NULL schedule");
    NEED(mode == HIOS_STAGE_STREAMS || mode == HIOS_STAGE_GROUPED || mode == HIOS_STAGE_DATAFLOW ||
             mode == HIOS_STAGE_AUTO,
         HIOS_E_INVALID, "unknown stage mode");
    NEED(!s->s->exec, HIOS_E_STATE, "set the stage mode before the first run");
    s->s->stage_mode = mode;
  });
}

hios_status hios_nccl_unique_id(void* id128) {
  return guard([&] {
    NEED(id128, HIOS_E_INVALID, "NULL id");
    hios::NcclUniqueId id;
    hios::nccl_unique_id(&id);
    memcpy(id128, &id, sizeof(id));
  });
}

hios_status hios_schedule_nccl_init(hios_schedule s, const void* id128, int32_t nranks, int32_t rank) {
  return guard([&] {
    NEED(s && id128 && nranks >= 1 && rank >= 0 && rank < nranks, HIOS_E_INVALID, "bad argument");
    auto& S = *s->s;
    NEED(!S.owner.empty(), HIOS_E_STATE, "NCCL transport: bind ranks first (hios_schedule_bind_rank)");
    NEED(S.rank == rank, HIOS_E_INVALID, "rank differs from hios_schedule_bind_rank's");
    NEED(S.transport == HIOS_TRANSPORT_NCCL, HIOS_E_STATE, "set HIOS_TRANSPORT_NCCL first");
    int dev = -1;
    for (int l = 0; l < S.M; ++l) {
      if (S.owner[l] != rank) continue;
      const int d = S.devices.empty() ? 0 : S.devices[l];
      NEED(dev < 0 || dev == d, HIOS_E_UNSUPPORTED, "NCCL transport: a rank's logical GPUs must share one device");
      dev = d;
    }
    auto& E = ensure_exec(S);
    NEED(!E.comm, HIOS_E_STATE, "NCCL already initialised");
    NEED(!E.captured, HIOS_E_STATE, "initialise NCCL before the first run");
    hios::NcclUniqueId id;
    memcpy(&id, id128, sizeof(id));
    E.comm = hios::nccl_comm_init(dev < 0 ? 0 : dev, id, nranks, rank);
  });
}

hios_status hios_schedule_transfers(hios_schedule s, int32_t* src_op, int32_t* dst_gpu, int32_t cap, int32_t* n) {
  return guard([&] {
    NEED(s && n, HIOS_E_INVALID, "NULL argument");
    auto t = hios::transfer_order(*s->s);
    *n = (int32_t)t.size();
    if (!src_op && !dst_gpu) return;
    NEED(src_op && dst_gpu && cap >= (int32_t)t.size(), HIOS_E_INVALID, "arrays too small");
    for (size_t i = 0; i < t.size(); ++i) {
      src_op[i] = t[i].first;
      dst_gpu[i] = t[i].second;
    }
  });
}

// blob: [int32 n][n x { int32 lgpu, cudaIpcMemHandle arena, cudaIpcMemHandle sync }]
hios_status hios_ipc_export(hios_schedule s, void* blob, size_t* len) {
  return guard([&] {
    NEED(s && len, HIOS_E_INVALID, "NULL argument");
    auto& E = ensure_exec(*s->s);
    if (!E.lowered) {
      E.plan();
      E.allocate();
    }
    std::vector<char> out(sizeof(int32_t));
    int32_t cnt = 0;
    for (int l = 0; l < E.M; ++l) {
      if (!E.lg[l].local) continue;
      cudaIpcMemHandle_t ha, hs;
      hios::ck(cudaSetDevice(E.lg[l].dev), "cudaSetDevice");
      hios::ck(cudaIpcGetMemHandle(&ha, E.lg[l].arena), "cudaIpcGetMemHandle");
      hios::ck(cudaIpcGetMemHandle(&hs, E.lg[l].sync), "cudaIpcGetMemHandle");
      int32_t id = l;
      size_t at = out.size();
      out.resize(at + sizeof(id) + 2 * sizeof(cudaIpcMemHandle_t));
      memcpy(&out[at], &id, sizeof(id));
      memcpy(&out[at + sizeof(id)], &ha, sizeof(ha));
      memcpy(&out[at + sizeof(id) + sizeof(ha)], &hs, sizeof(hs));
      ++cnt;
    }
    memcpy(out.data(), &cnt, sizeof(cnt));
    if (!blob || *len < out.size()) {
      *len = out.size();
      NEED(blob == nullptr, HIOS_E_INVALID, "blob too small");
      return;
    }
    memcpy(blob, out.data(), out.size());
    *len = out.size();
  });
}

hios_status hios_ipc_import(hios_schedule s, int32_t rank, const void* blob, size_t len) {
  return guard([&] {
    NEED(s && blob && len >= sizeof(int32_t), HIOS_E_INVALID, "bad blob");
    auto& E = ensure_exec(*s->s);
    NEED(E.lowered, HIOS_E_STATE, "export before import");
    const char* p = (const char*)blob;
    int32_t cnt;
    memcpy(&cnt, p, sizeof(cnt));
    size_t at = sizeof(cnt);
    for (int i = 0; i < cnt; ++i) {
      NEED(at + sizeof(int32_t) + 2 * sizeof(cudaIpcMemHandle_t) <= len, HIOS_E_INVALID, "truncated blob");
      int32_t l;
      cudaIpcMemHandle_t ha, hs;
      memcpy(&l, p + at, sizeof(l));
      memcpy(&ha, p + at + sizeof(l), sizeof(ha));
      memcpy(&hs, p + at + sizeof(l) + sizeof(ha), sizeof(hs));
      at += sizeof(l) + 2 * sizeof(cudaIpcMemHandle_t);
      NEED(l >= 0 && l < E.M, HIOS_E_INVALID, "bad logical GPU in blob");
      NEED(!s->s->owner.empty() && s->s->owner[l] == rank, HIOS_E_INVALID, "blob GPU not owned by rank");
      auto& L = E.lg[l];
      if (L.local || L.ipc_mapped) continue;
      // the mapping is made in the context of this rank's device: rank mode
      // supports one device per rank (its logical GPUs may alias it), so the
      // pointer is valid for every local kernel
      int dev = -1;
      for (auto& x : E.lg)
        if (x.local) {
          NEED(dev < 0 || dev == x.dev, HIOS_E_UNSUPPORTED,
               "rank mode: a rank's logical GPUs must share one device (IPC maps are per device)");
          dev = x.dev;
        }
      NEED(dev >= 0, HIOS_E_STATE, "no local GPU");
      hios::ck(cudaSetDevice(dev), "cudaSetDevice");
      void* a = nullptr;
      void* sy = nullptr;
      hios::ck(cudaIpcOpenMemHandle(&a, ha, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
      hios::ck(cudaIpcOpenMemHandle(&sy, hs, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
      L.arena = (char*)a;
      L.sync = (unsigned*)sy;
      L.ipc_mapped = true;
    }
  });
}

hios_status hios_output_numel(hios_schedule s, int64_t* n) {
  return guard([&] {
    NEED(s && n, HIOS_E_INVALID, "NULL argument");
    auto& o = s->s->g->ops[s->s->g->sink_op];
    *n = (int64_t)o.C * o.H * o.W;
  });
}

static void check_remote_mapped(hios::Executor& E) {
  for (int l = 0; l < E.M; ++l)
    NEED(E.lg[l].local || E.lg[l].ipc_mapped, HIOS_E_STATE,
         "rank mode: import every other rank's IPC blob before running");
}

hios_status hios_run_device(hios_schedule s, const void* d_in, void* d_out, void* stream) {
  return guard([&] {
    NEED(s, HIOS_E_INVALID, "NULL schedule");
    auto& E = ensure_exec(*s->s);
    if (!s->s->owner.empty()) {
      NEED(E.lowered, HIOS_E_STATE, "rank mode: hios_ipc_export/import first");
      check_remote_mapped(E);
    }
    E.run_device(d_in, d_out, (cudaStream_t)stream, false);
  });
}

hios_status hios_run_timed(hios_schedule s, const void* d_in, void* d_out, void* stream, int64_t* op_ns) {
  return guard([&] {
    NEED(s, HIOS_E_INVALID, "NULL schedule");
    auto& E = ensure_exec(*s->s);
    if (!s->s->owner.empty()) check_remote_mapped(E);
    E.run_device(d_in, d_out, (cudaStream_t)stream, true);
    if (op_ns) {
      if (stream) hios::ck(cudaStreamSynchronize((cudaStream_t)stream), "sync");
      for (int v = 0; v < E.g.n; ++v) {
        op_ns[v] = -1;
        const int l = s->s->gpu_of[v];
        if (!E.lg[l].local || !E.op_ev0[v]) continue;
        float ms = 0;
        hios::ck(cudaEventElapsedTime(&ms, E.op_ev0[v], E.op_ev1[v]), "elapsed");
        op_ns[v] = (int64_t)(ms * 1e6);
      }
    }
  });
}

hios_status hios_run(hios_schedule s, const float* input, float* output) {
  return guard([&] {
    NEED(s, HIOS_E_INVALID, "NULL schedule");
    auto& S = *s->s;
    auto& E = ensure_exec(S);
    auto& G = *S.g;
    if (!S.owner.empty()) {
      NEED(E.lowered, HIOS_E_STATE, "rank mode: hios_ipc_export/import first");
      check_remote_mapped(E);
    }
    if (!E.lowered) {
      E.plan();
      E.allocate();
    }
    const int li = S.gpu_of[G.input_op], ls = S.gpu_of[G.sink_op];
    const size_t nin = (size_t)G.in_c * G.in_h * G.in_w;
    const auto& so = G.ops[G.sink_op];
    const size_t nout = (size_t)so.C * so.H * so.W;
    if (E.lg[li].local) {
      NEED(input, HIOS_E_INVALID, "input is NULL");
      hios::ck(cudaSetDevice(E.lg[li].dev), "cudaSetDevice");
      if (!E.d_in_stage) hios::ck(cudaMalloc(&E.d_in_stage, nin * sizeof(float)), "cudaMalloc");
      hios::ck(cudaMemcpy(E.d_in_stage, input, nin * sizeof(float), cudaMemcpyHostToDevice), "H2D input");
    }
    if (E.lg[ls].local) {
      NEED(output, HIOS_E_INVALID, "output is NULL");
      hios::ck(cudaSetDevice(E.lg[ls].dev), "cudaSetDevice");
      if (!E.d_out_stage) hios::ck(cudaMalloc(&E.d_out_stage, nout * sizeof(float)), "cudaMalloc");
    }
    E.run_device(E.lg[li].local ? E.d_in_stage : nullptr, E.lg[ls].local ? E.d_out_stage : nullptr, nullptr,
                 false);
    if (E.lg[ls].local) {
      hios::ck(cudaSetDevice(E.lg[ls].dev), "cudaSetDevice");
      hios::ck(cudaMemcpy(output, E.d_out_stage, nout * sizeof(float), cudaMemcpyDeviceToHost), "D2H output");
    }
  });
}

hios_status hios_read_op_output(hios_schedule s, int32_t op, float* host, int64_t n) {
  return guard([&] {
    NEED(s && host && op >= 0 && op < s->s->g->n, HIOS_E_INVALID, "bad argument");
    NEED(s->s->exec && s->s->exec->captured, HIOS_E_STATE, "run first");
    s->s->exec->read_output(op, host, n);
  });
}

hios_status hios_time_ops(hios_schedule s, int32_t reps, int64_t flush_bytes, int64_t* op_ns) {
  return guard([&] {
    NEED(s && op_ns && reps >= 1 && flush_bytes >= 0, HIOS_E_INVALID, "bad argument");
    auto& E = ensure_exec(*s->s);
    if (!s->s->owner.empty()) check_remote_mapped(E);
    E.time_ops(reps, flush_bytes, op_ns);
  });
}

hios_status hios_schedule_stage_mode_used(hios_schedule s, int32_t* mode) {
  return guard([&] {
    NEED(s && mode, HIOS_E_INVALID, "NULL argument");
    NEED(s->s->exec && s->s->exec->captured, HIOS_E_STATE, "run first");
    *mode = s->s->exec->mode_used;
  });
}

hios_status hios_op_output_relu(hios_schedule s, int32_t op, int32_t* relu) {
  return guard([&] {
    NEED(s && relu && op >= 0 && op < s->s->g->n, HIOS_E_INVALID, "bad argument");
    NEED(s->s->exec && s->s->exec->captured, HIOS_E_STATE, "run first");
    *relu = s->s->exec->relu_out[op] ? 1 : 0;
  });
}

hios_status hios_op_plan(hios_schedule s, int32_t op, int32_t solo, int32_t* plan) {
  return guard([&] {
    NEED(s && plan && op >= 0 && op < s->s->g->n, HIOS_E_INVALID, "bad argument");
    NEED(s->s->exec && s->s->exec->captured, HIOS_E_STATE, "run first");
    const hios::OpExec& x = s->s->exec->ox[op];
    for (int i = 0; i < 8; ++i) plan[i] = solo ? x.plan_solo[i] : x.plan[i];
  });
}

hios_status hios_kernel_count(hios_schedule s, int64_t* n) {
  return guard([&] {
    NEED(s && n, HIOS_E_INVALID, "NULL argument");
    NEED(s->s->exec && s->s->exec->captured, HIOS_E_STATE, "run first");
    int64_t extra = 0;
    auto& S = *s->s;
    if (S.exec->lg[S.gpu_of[S.g->input_op]].local) ++extra;  // input conversion
    if (S.exec->lg[S.gpu_of[S.g->sink_op]].local) ++extra;   // output conversion
    *n = S.exec->kernels_per_run + extra;
  });
}

}  // extern "C"
