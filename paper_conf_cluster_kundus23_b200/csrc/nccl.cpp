// nccl.cpp -- the NCCL send/recv fallback transport of the cross-GPU edges
// ("inter-GPU data transfer based on ... NCCL might be able to
// hide the launching time of succeeding CUDA kernels"; the paper's own engine
// used CUDA-aware MPI).  libnccl.so.2 is loaded at run time so the
// library has no link-time NCCL dependency; only the handful of calls the
// transport needs are resolved.
//
// transfer_order() is the global order every process posts its sends and
// receives in: ascending position of the producer's stage in a topological
// order of the stage DAG (per-GPU stage order + data edges), ties by producer
// op id, then consumer GPU.  Any transfer a stage X depends on (directly or
// through earlier stages of X's GPU) has a producer stage that precedes X in
// that order, so when every GPU's communication stream walks the list in
// order, each send/recv pair can match without waiting on a later one.
#include <dlfcn.h>

#include <algorithm>
#include <cstdlib>
#include <queue>
#include <set>

#include "exec.h"

namespace hios {

struct NcclApi {
  bool ok = false;
  std::string err;
  int (*GetUniqueId)(NcclUniqueId*) = nullptr;
  int (*CommInitRank)(NcclComm*, int, NcclUniqueId, int) = nullptr;
  int (*CommDestroy)(NcclComm) = nullptr;
  int (*Send)(const void*, size_t, int, int, NcclComm, cudaStream_t) = nullptr;
  int (*Recv)(void*, size_t, int, int, NcclComm, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(int) = nullptr;
};

static NcclApi& nccl() {
  static NcclApi api;
  static bool tried = false;
  if (tried) return api;
  tried = true;
  const char* path = getenv("HIOS_NCCL_LIB");
  void* h = dlopen(path ? path : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    api.err = std::string("cannot load ") + (path ? path : "libnccl.so.2") + ": " + dlerror();
    return api;
  }
  auto sym = [&](const char* n) {
    void* p = dlsym(h, n);
    if (!p) api.err = std::string("missing symbol ") + n;
    return p;
  };
  api.GetUniqueId = (int (*)(NcclUniqueId*))sym("ncclGetUniqueId");
  api.CommInitRank = (int (*)(NcclComm*, int, NcclUniqueId, int))sym("ncclCommInitRank");
  api.CommDestroy = (int (*)(NcclComm))sym("ncclCommDestroy");
  api.Send = (int (*)(const void*, size_t, int, int, NcclComm, cudaStream_t))sym("ncclSend");
  api.Recv = (int (*)(void*, size_t, int, int, NcclComm, cudaStream_t))sym("ncclRecv");
  api.GetErrorString = (const char* (*)(int))sym("ncclGetErrorString");
  api.ok = api.err.empty();
  return api;
}

static void nck(int r, const char* what) {
  if (r != 0) {
    const char* m = nccl().GetErrorString ? nccl().GetErrorString(r) : "?";
    fail(HIOS_E_NCCL, std::string(what) + ": " + m);
  }
}

constexpr int kNcclUint8 = 1;  // ncclDataType_t ncclUint8: transfers are byte counts

void nccl_unique_id(NcclUniqueId* id) {
  NcclApi& a = nccl();
  if (!a.ok) fail(HIOS_E_NCCL, a.err);
  nck(a.GetUniqueId(id), "ncclGetUniqueId");
}

NcclComm nccl_comm_init(int dev, const NcclUniqueId& id, int nranks, int rank) {
  NcclApi& a = nccl();
  if (!a.ok) fail(HIOS_E_NCCL, a.err);
  ck(cudaSetDevice(dev), "cudaSetDevice");
  NcclComm c = nullptr;
  nck(a.CommInitRank(&c, nranks, id, rank), "ncclCommInitRank");
  return c;
}

void nccl_comm_destroy(NcclComm c) {
  if (c && nccl().ok) nccl().CommDestroy(c);
}

void nccl_send(const void* buf, size_t bytes, int peer, NcclComm c, cudaStream_t st) {
  nck(nccl().Send(buf, bytes, kNcclUint8, peer, c, st), "ncclSend");
}

void nccl_recv(void* buf, size_t bytes, int peer, NcclComm c, cudaStream_t st) {
  nck(nccl().Recv(buf, bytes, kNcclUint8, peer, c, st), "ncclRecv");
}

std::vector<std::vector<int>> stage_ranks(const Schedule& s) {
  const Graph& g = *s.g;
  // stages as nodes: id = offset[gpu] + stage
  std::vector<int> off(s.M + 1, 0);
  for (int i = 0; i < s.M; ++i) off[i + 1] = off[i] + (int)s.Q[i].size();
  const int ns = off[s.M];
  std::vector<std::set<int>> succ(ns);
  std::vector<int> indeg(ns, 0);
  auto node = [&](int v) { return off[s.gpu_of[v]] + s.stage_of[v]; };
  for (int i = 0; i < s.M; ++i)
    for (int j = 0; j + 1 < (int)s.Q[i].size(); ++j) succ[off[i] + j].insert(off[i] + j + 1);
  for (const Edge& e : g.edges) {
    const int a = node(e.src), b = node(e.dst);
    if (a != b) succ[a].insert(b);
  }
  for (int a = 0; a < ns; ++a)
    for (int b : succ[a]) ++indeg[b];
  std::priority_queue<int, std::vector<int>, std::greater<int>> q;
  for (int a = 0; a < ns; ++a)
    if (!indeg[a]) q.push(a);
  std::vector<int> rank(ns, -1);
  int r = 0;
  while (!q.empty()) {
    const int a = q.top();
    q.pop();
    rank[a] = r++;
    for (int b : succ[a])
      if (--indeg[b] == 0) q.push(b);
  }
  if (r != ns) fail(HIOS_E_CYCLE, "stage graph has a cycle");
  std::vector<std::vector<int>> out(s.M);
  for (int i = 0; i < s.M; ++i)
    for (int j = 0; j < (int)s.Q[i].size(); ++j) out[i].push_back(rank[off[i] + j]);
  return out;
}

std::vector<std::pair<int, int>> transfer_order(const Schedule& s) {
  const Graph& g = *s.g;
  const std::vector<std::vector<int>> rk = stage_ranks(s);
  auto node_rank = [&](int v) { return rk[s.gpu_of[v]][s.stage_of[v]]; };
  std::vector<std::tuple<int, int, int>> t;
  for (int u = 0; u < g.n; ++u) {
    std::set<int> dst;
    for (int e : g.ops[u].out_edges) {
      const int l = s.gpu_of[g.edges[e].dst];
      if (l != s.gpu_of[u]) dst.insert(l);
    }
    for (int l : dst) t.emplace_back(node_rank(u), u, l);
  }
  std::sort(t.begin(), t.end());
  std::vector<std::pair<int, int>> out;
  for (auto& x : t) out.push_back({std::get<1>(x), std::get<2>(x)});
  return out;
}

}  // namespace hios
