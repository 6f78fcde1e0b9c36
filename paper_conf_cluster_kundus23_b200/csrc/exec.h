// exec.h -- per-GPU stage executor.
#pragma once
#include <functional>
#include <map>
#include <set>
#include <vector>

#include "internal.h"
#include "kernels.cuh"

namespace hios {

// NCCL transport (nccl.cpp; libnccl.so.2 loaded at run time)
struct NcclUniqueId { char internal[128]; };
typedef struct ncclComm* NcclComm;
void nccl_unique_id(NcclUniqueId* id);
NcclComm nccl_comm_init(int dev, const NcclUniqueId& id, int nranks, int rank);
void nccl_comm_destroy(NcclComm c);
void nccl_send(const void* buf, size_t bytes, int peer, NcclComm c, cudaStream_t st);
void nccl_recv(void* buf, size_t bytes, int peer, NcclComm c, cudaStream_t st);
// global order of the (producer op, consumer logical GPU) transfers
std::vector<std::pair<int, int>> transfer_order(const Schedule& s);
// position of every stage (gpu, j) in one topological order of the stage DAG
std::vector<std::vector<int>> stage_ranks(const Schedule& s);

// how one (producer, consumer GPU) edge is carried
enum DeliverMode { DM_FUSED = 0, DM_PUSH = 1, DM_COPY = 2, DM_NCCL = 3 };
struct Remote {
  int gpu;   // consumer logical GPU
  int mode;  // DeliverMode
};

struct Loc {
  int64_t off = -1;  // byte offset in the owning logical GPU's arena
  int ldc = 0;       // pixel stride in elements
};

struct OpExec {
  // device weights (home logical GPU)
  void* w = nullptr;       // conv / linear weights (T) or sepconv pw weights per rep
  std::vector<void*> pw;   // sepconv: per-rep pointwise weights
  std::vector<float*> dw;  // sepconv: per-rep depthwise weights [RS][C] fp32
  std::vector<float*> scale, shift;
  float* w_small = nullptr;  // direct small-C conv weights [K][R][S][C] fp32
  float* bias = nullptr;
  int ldw = 0;
  // sepconv scratch (arena offsets)
  int64_t dwbuf = -1, midbuf = -1;
  // pre-ReLU conv whose producer is remote / the input: its ReLU'd input copy
  int64_t relubuf = -1;
  int relu_ldc = 0;
  int dw_ldc = 0, mid_ldc = 0;
  // stride-2 small-C stem (bf16): space-to-depth copy of the input (arena offset)
  // a conv whose weights are zero at every tap but (tap_r, tap_s) (NASNet's
  // factorized-reduction path 2: a shifted, strided 1x1 conv written as a
  // 3x3 conv): x.w holds that tap only and the conv runs as 1x1 on the input
  // shifted by the tap (padding ph - tap_r * dh, pw - tap_s * dw)
  int tap_r = -1, tap_s = -1;
  int64_t s2dbuf = -1;
  int s2d_ldc = 0;
  // s2d stem with its S' taps packed into one 64-element K row (overlapping
  // 4-pixel windows of the s2d tensor; weights W''[k][r'][s'*16 + ch])
  void* w_pack = nullptr;
  // remote deliveries of this op's output
  std::vector<Remote> remote;
  std::function<void(cudaStream_t)> run;  // enqueue the op's kernels (incl. fused out2)
  int n_kernels = 0;
  // the same op configured to run alone (a singleton stage / t(v) profiling):
  // tap-mode convs take narrower N tiles there (more CTAs); empty = run
  std::function<void(cudaStream_t)> run_solo;
  int n_kernels_solo = 0;
  // tcgen05 conv tile plan (hios_op_plan): {A mode (1 tap, 2 halo, 3 vgrid
  // halo), n_tile, output tiles, epilogue mode, 256-bit stores, rows per
  // tile, stages, K-steps per stage}; [0] = 0 for any other op / path
  int plan[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  int plan_solo[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  // a plain tcgen05 conv (one launch, group-context plan): its descriptor for
  // the stage's grouped launch (conv_tc_group_kernel); empty otherwise
  std::vector<ConvTcOp> tc;
  size_t tc_smem = 0;
  // profiler only: one extra epilogue destination (the t(u, v) probe of C15)
  char* probe_out = nullptr;
  int probe_ldc = 0;
};

struct LGpu {
  int dev = 0;
  bool local = true;
  std::vector<cudaStream_t> streams;
  cudaEvent_t ev_fork = nullptr;
  std::vector<cudaEvent_t> ev_join;
  cudaEvent_t ev_start = nullptr, ev_done = nullptr;
  cudaGraphExec_t gexec = nullptr, gexec_timed = nullptr;
  // HIOS_STAGE_AUTO: the other executor variant's graphs until the first run
  // has measured both (then the faster one is gexec / gexec_timed)
  cudaGraphExec_t gexec_alt = nullptr, gexec_timed_alt = nullptr;
  char* arena = nullptr;       // local: owned; remote (rank mode): IPC-mapped
  size_t arena_bytes = 0;
  unsigned* sync = nullptr;    // [0] epoch, [1 .. 1+M) acks, then flags
  size_t sync_words = 0;
  std::vector<void*> allocs;   // weights etc. (owned)
  bool ipc_mapped = false;
  cudaStream_t comm = nullptr;  // NCCL transport: send/recv stream
  int num_sms = 148;             // cudaDevAttrMultiProcessorCount
};

// one NCCL transfer of the global order, as this process sees it
struct NcclXfer {
  int u = -1, src = -1, dst = -1;  // producer op, producer / consumer logical GPU
  int64_t send_off = -1, recv_off = -1;  // staging (packed H*W*C) or -1: direct
  size_t bytes = 0;
  cudaEvent_t ev_ready = nullptr;  // producer: op u finished (on its GPU)
  cudaEvent_t ev_recv = nullptr;   // consumer: data landed
};

struct Executor {
  Schedule& s;
  Graph& g;
  int M;
  int esz;  // element size
  std::vector<LGpu> lg;
  std::vector<std::vector<Loc>> loc;   // loc[op][lgpu]
  std::map<int64_t, Loc> relu_loc;     // (producer * M + lgpu) -> ReLU'd copy for pre-ReLU convs
  std::vector<char> inplace;           // per edge: producer writes into the concat slice
  // per op: every consumer applies ReLU to this output first (pre-ReLU convs /
  // separable convs, single-input ReLU adds, or a concat whose own consumers
  // all do), so the op stores its output already ReLU'd and the consumers
  // read it without a ReLU'd copy (ReLU(bf16(y)) = bf16(ReLU(y)): exact)
  std::vector<char> relu_out;
  std::vector<char> relu_copy_in;  // per edge: the ReLU'd concat copies this raw input's slice
  std::vector<OpExec> ox;
  std::vector<std::vector<int>> flag_index;  // [op][lgpu] flag slot on that lgpu (-1 none)
  int n_streams = 1;
  int transport = HIOS_TRANSPORT_PEER;  // cross-GPU edge transport (hios_schedule_transport)
  NcclComm comm = nullptr;              // NCCL transport: this rank's communicator
  std::vector<NcclXfer> xfers;          // NCCL transfers in the global order
  int cur_lgpu = 0;  // logical GPU whose closures are being built
  bool lowered = false, captured = false;
  int64_t kernels_per_run = 0;
  // timed-graph events: per op (start, end) on its home lgpu
  std::vector<cudaEvent_t> op_ev0, op_ev1;
  // staging for hios_run (host pointers)
  float* d_in_stage = nullptr;
  float* d_out_stage = nullptr;

  explicit Executor(Schedule& sch);
  ~Executor();
  void plan();             // locations, flags (host only)
  void allocate();         // arenas, sync words, weights (local lgpus)
  void build_closures();   // per-op kernel launchers
  void build_op_closures(int v);  // op v's launchers (group and solo configs)
  void capture();          // per-lgpu CUDA graphs
  void run_device(const void* d_in, void* d_out, cudaStream_t user, bool timed);
  char* ptr(int lgpu, int64_t off) const { return lg[lgpu].arena + off; }
  bool is_local(int l) const { return lg[l].local; }
  void read_output(int op, float* host, int64_t n);
  // CUDA graph per device: its local logical GPUs' stage programs
  void capture_device(const std::vector<int>& ls, bool timed);
  std::map<int, std::vector<int>> graphs_by_dev;  // device -> local lgpus (first = owner)
  std::vector<int> graph_of;                      // lgpu -> owner lgpu of its graph (-1 remote)
  std::map<int64_t, cudaEvent_t> edge_ev;         // (u * M + consumer lgpu) -> same-graph edge event
  std::set<int> cur_graph;
  bool same_graph(int a, int b) const {
    return a >= 0 && b >= 0 && a < (int)graph_of.size() && b < (int)graph_of.size() && graph_of[a] >= 0 &&
           graph_of[a] == graph_of[b];
  }
  cudaEvent_t edge_event(int u, int d);
  // each local op's kernels alone, L2 flushed, as configured in Q (hios_time_ops)
  void time_ops(int reps, int64_t flush_bytes, int64_t* op_ns);
  // one stage S of logical GPU l: its plain tcgen05 convs as ONE grouped
  // launch on s0 with an explicit SM partition, the other ops forked onto
  // streams 1.. (or every op on its own stream: group == false); post(v, st)
  // runs after op v on the stream v ran on
  // (lane != nullptr: the ops run on that stream instead of stream 0;
  // singleton: a one-op stage takes the op's solo plan)
  void enqueue_stage(int l, const std::vector<int>& S, bool timed, int64_t& nk,
                     const std::function<void(int, cudaStream_t)>& post, cudaStream_t lane = nullptr,
                     bool singleton = true);
  bool group_convs = false;  // hios_schedule_stage_mode
  bool dataflow = false;     // HIOS_STAGE_DATAFLOW: per-op input waits instead of stage joins
  bool auto_pending = false; // HIOS_STAGE_AUTO: streams vs dataflow not measured yet
  int mode_used = 0;         // the stage mode the graphs execute (hios_schedule_stage_mode_used)
  void choose_variant();     // HIOS_STAGE_AUTO: time both variants' graphs, keep the faster
  std::vector<cudaEvent_t> done_ev;  // dataflow: op v finished on its lane
  std::vector<int> lane_of;          // dataflow: the lane (stream index) op v ran on
};

void ck(cudaError_t e, const char* what);

}  // namespace hios
