// profile.cu -- hios_profile ("the scheduling
// time includes the time used to measure the execution time of each single
// operator and each group of parallel operators, the communication time of
// each possible data transfer between GPUs ...").
//
//   t(v)    median of `reps` CUDA-event timings of op v's kernels alone
//   t(u,v)  SURVEY C15: for ops whose epilogue stores straight into the
//           consumer GPU's buffer (conv / sepconv / pools / add), the
//           incremental cost of that extra destination, t(u fused) - t(u);
//           for the others the time of the peer-store push kernel; plus one
//           flag release/acquire pair; the same for every edge leaving u
//   t(S)    measured on demand (Profiler::measure_group): the ops of S forked
//           onto |S| streams from one event and joined, median of reps
#include <algorithm>

#include "exec.h"

namespace hios {

class ProfilerImpl : public Profiler {
 public:
  Schedule sched;
  int reps = 10;
  int peer_dev = -1;
  explicit ProfilerImpl(std::shared_ptr<Graph> g) { sched.g = g; }
  ~ProfilerImpl() override {}

  Executor& ex() { return *sched.exec; }

  // Device time of fn as it runs inside the executor's CUDA graphs: `reps`
  // back-to-back copies are captured into one graph, replayed (warm-up), then
  // timed with events; median over 3 replays / reps.  Host launch latency is
  // excluded, the in-graph kernel-to-kernel gaps are included.
  int64_t time_ns(const std::function<void(cudaStream_t)>& fn, cudaStream_t st) {
    cudaGraph_t graph;
    ck(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed), "profile capture");
    for (int i = 0; i < reps; ++i) fn(st);
    ck(cudaStreamEndCapture(st, &graph), "profile capture end");
    cudaGraphExec_t ge;
    ck(cudaGraphInstantiate(&ge, graph, 0), "profile instantiate");
    cudaGraphDestroy(graph);
    cudaEvent_t a, b;
    ck(cudaEventCreate(&a), "event");
    ck(cudaEventCreate(&b), "event");
    ck(cudaGraphLaunch(ge, st), "profile launch");
    std::vector<float> ms;
    for (int i = 0; i < 3; ++i) {
      ck(cudaEventRecord(a, st), "record");
      ck(cudaGraphLaunch(ge, st), "profile launch");
      ck(cudaEventRecord(b, st), "record");
      ck(cudaEventSynchronize(b), "sync");
      float t = 0;
      ck(cudaEventElapsedTime(&t, a, b), "elapsed");
      ms.push_back(t / reps);
    }
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaGraphExecDestroy(ge);
    std::sort(ms.begin(), ms.end());
    return (int64_t)(ms[1] * 1e6);
  }

  int64_t measure_group(Graph& g, const std::vector<int>& S) override {
    Executor& E = ex();
    LGpu& L = E.lg[0];
    ck(cudaSetDevice(L.dev), "cudaSetDevice");
    if ((int)S.size() > E.n_streams) fail(HIOS_E_UNSUPPORTED, "group larger than the profiler's streams");
    // exactly as the executor runs a stage (grouped conv launch + forked
    // streams for the rest, Executor::enqueue_stage), on streams[0]
    auto fn = [&](cudaStream_t s0) {
      (void)s0;
      int64_t nk = 0;
      E.enqueue_stage(0, S, false, nk, [](int, cudaStream_t) {});
    };
    (void)g;
    return time_ns(fn, L.streams[0]);
  }
};

std::shared_ptr<Profiler> run_profile(std::shared_ptr<Graph> G, const int32_t* devices, int32_t n_devices,
                                      int32_t reps) {
  Graph& g = *G;
  // non-owning alias: the profiler lives inside the graph
  auto impl = std::make_shared<ProfilerImpl>(std::shared_ptr<Graph>(std::shared_ptr<Graph>(), &g));
  impl->reps = std::max(3, reps);
  Schedule& s = impl->sched;
  s.M = 1;
  s.w = 8;
  s.Q.assign(1, {});
  for (int v : g.topo) s.Q[0].push_back({v});
  s.Q[0][0].reserve(1);
  s.gpu_of.assign(g.n, 0);
  s.stage_of.resize(g.n);
  for (int k = 0; k < g.n; ++k) s.stage_of[g.topo[k]] = k;
  const int dev0 = n_devices > 0 ? devices[0] : 0;
  s.devices = {dev0};
  s.exec.reset(new Executor(s));
  Executor& E = *s.exec;
  E.n_streams = 8;
  E.plan();
  E.allocate();
  E.build_closures();
  LGpu& L = E.lg[0];
  ck(cudaSetDevice(L.dev), "cudaSetDevice");
  cudaStream_t st = L.streams[0];
  // realistic activations: a constant 0.5 input, then every op once in topological order
  {
    const size_t n = (size_t)g.in_c * g.in_h * g.in_w;
    std::vector<float> h(n, 0.5f);
    float* d = nullptr;
    ck(cudaMalloc(&d, n * sizeof(float)), "cudaMalloc");
    ck(cudaMemcpy(d, h.data(), n * sizeof(float), cudaMemcpyHostToDevice), "H2D");
    const Loc& lc = E.loc[g.input_op][0];
    if (g.dtype == HIOS_BF16) launch_input<bf16>(d, g.in_c, g.in_h, g.in_w, (bf16*)E.ptr(0, lc.off), lc.ldc, st);
    else launch_input<float>(d, g.in_c, g.in_h, g.in_w, (float*)E.ptr(0, lc.off), lc.ldc, st);
    for (int v : g.topo) E.ox[v].run(st);
    ck(cudaStreamSynchronize(st), "profile warm-up");
    // t(input) = the layout conversion of the input
    const int vin = g.input_op;
    auto fin = [&](cudaStream_t s2) {
      if (g.dtype == HIOS_BF16) launch_input<bf16>(d, g.in_c, g.in_h, g.in_w, (bf16*)E.ptr(0, lc.off), lc.ldc, s2);
      else launch_input<float>(d, g.in_c, g.in_h, g.in_w, (float*)E.ptr(0, lc.off), lc.ldc, s2);
    };
    g.ops[vin].cost = impl->time_ns(fin, st);
    cudaFree(d);
  }
  for (int v : g.topo) {
    if (v == g.input_op) continue;
    g.ops[v].cost = impl->time_ns(E.ox[v].run_solo ? E.ox[v].run_solo : E.ox[v].run, st);
  }
  // t(u, v): push of u's output into a buffer on the peer device (or a second buffer here)
  const int peer = n_devices > 1 ? devices[1] : dev0;
  size_t max_bytes = 16;
  for (auto& o : g.ops) max_bytes = std::max(max_bytes, (size_t)o.H * o.W * ((o.C + 7) / 8 * 8) * E.esz);
  void* dst = nullptr;
  unsigned* flag = nullptr;
  ck(cudaSetDevice(peer), "cudaSetDevice");
  ck(cudaMalloc(&dst, max_bytes), "cudaMalloc");
  ck(cudaMalloc(&flag, 64), "cudaMalloc");
  ck(cudaMemset(flag, 0, 64), "memset");
  if (peer != dev0) {
    ck(cudaSetDevice(dev0), "cudaSetDevice");
    cudaError_t e = cudaDeviceEnablePeerAccess(peer, 0);
    if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) ck(e, "peer access");
    cudaGetLastError();
  }
  ck(cudaSetDevice(dev0), "cudaSetDevice");
  unsigned* epoch = L.sync;
  auto fsync = [&](cudaStream_t s2) {
    launch_epoch(epoch, s2);
    launch_signal(epoch, flag, s2);
    launch_wait(epoch, flag, 0, s2);
  };
  const int64_t t_sync = impl->time_ns(fsync, st);
  std::vector<int64_t> push(g.n, -1);
  for (int u = 0; u < g.n; ++u) {
    if (g.ops[u].out_edges.empty()) continue;
    const Op& o = g.ops[u];
    const Loc& lc = E.loc[u][0];
    // C15: ops whose epilogue can store straight into the consumer GPU's
    // buffer (conv / sepconv / pools / add) pay only the INCREMENTAL cost of
    // that extra destination: t(u with the remote store) - t(u), >= 0
    const bool fusable = o.kind == HIOS_OP_CONV || o.kind == HIOS_OP_SEPCONV || o.kind == HIOS_OP_MAXPOOL ||
                         o.kind == HIOS_OP_AVGPOOL || o.kind == HIOS_OP_ADD;
    if (fusable && u != g.input_op) {
      OpExec& x = E.ox[u];
      x.probe_out = (char*)dst;
      x.probe_ldc = (o.C + 7) / 8 * 8;
      E.build_op_closures(u);
      const int64_t t_fused = impl->time_ns(x.run_solo ? x.run_solo : x.run, st);
      x.probe_out = nullptr;
      E.build_op_closures(u);
      push[u] = std::max<int64_t>(0, t_fused - g.ops[u].cost);
      continue;
    }
    std::function<void(cudaStream_t)> f;
    if (g.dtype == HIOS_BF16) {
      CopyArgs<bf16> c{(const bf16*)E.ptr(0, lc.off), lc.ldc, o.H * o.W, o.C, (bf16*)dst, (o.C + 7) / 8 * 8};
      f = [c](cudaStream_t s2) { launch_copy<bf16>(c, s2); };
    } else {
      CopyArgs<float> c{(const float*)E.ptr(0, lc.off), lc.ldc, o.H * o.W, o.C, (float*)dst, (o.C + 7) / 8 * 8};
      f = [c](cudaStream_t s2) { launch_copy<float>(c, s2); };
    }
    push[u] = impl->time_ns(f, st);
  }
  for (auto& e : g.edges) e.cost = push[e.src] + t_sync;
  ck(cudaSetDevice(peer), "cudaSetDevice");
  cudaFree(dst);
  cudaFree(flag);
  ck(cudaSetDevice(dev0), "cudaSetDevice");
  g.group_cost.clear();
  return impl;
}

}  // namespace hios
