// exec.cu -- lowering of a schedule Q to per-GPU stage programs and
// their replay as CUDA graphs.
//
//   * each logical GPU i executes Q_i stage by stage; the ops of one
//     stage fork onto up to w streams and join before the next stage
//   * every op output has a location on each logical GPU that consumes it;
//     a producer writes straight into the channel slice of a consumer concat
//     (zero-copy concat) -- on its own GPU or, for a cross-GPU edge, in the
//     consumer GPU's memory over NVLink (fused into the epilogue for conv /
//     pool / add, else a peer-store push kernel), then releases an epoch flag
//   * a stage waits device-side (acquire spin on the flag) for its remote
//     inputs: no host round trip between a transfer and the next kernel,
//     which is what the paper's MPI engine lacked
//   * stages of different GPUs are not synchronised otherwise
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <chrono>
#include <cstring>
#include <numeric>
#include <set>

#include "exec.h"

namespace hios {

// Stride-2 stems with <= 4 input channels on the tensor-core path (bf16):
// space-to-depth turns conv(R x S, stride 2, pad p) over C channels into
// conv(ceil(R/2) x ceil(S/2), stride 1, pad 0) over 4C channels of
//   X'[i][j][(a*2+b)*C + c] = X[2i+a-p][2j+b-p][c]      (zero outside X),
// with W'[k][r'][s'][(a*2+b)*C + c] = W[k][c][2r'+a][2s'+b] (zero past R, S).
// Every product of the original sum appears exactly once; K per tap is one
// K=16 MMA slice (4C <= 16) instead of a 64-channel chunk that is 95 % zero,
// and stride 1 lets the conv run in halo mode.
// 3x3 stride-2 stems over 3 channels with <= 40 outputs take the direct
// CUDA-core kernel (misc.cu conv_stem3_kernel; weights in the parameter bank):
// measured on B200, Inception Conv2d_1a at 4096^2 s2d + tcgen05 ~331 us,
// smem-weight CUDA-core kernel ~380 us (tools/stem_micro.py).  HIOS_NOSTEM3=1
// restores the s2d path.
static bool stem3_conv(const Op& o) {
  return o.kind == HIOS_OP_CONV && o.in_c == 3 && o.kh == 3 && o.kw == 3 && o.sh == 2 && o.sw == 2 &&
         o.dh == 1 && o.dw == 1 && o.out_c <= kStem3MaxK;
}
static bool s2d_conv(const Op& o) {
  return o.kind == HIOS_OP_CONV && !stem3_conv(o) && o.in_c <= 4 && o.sh == 2 && o.sw == 2 && o.dh == 1 && o.dw == 1 &&
         o.kh * o.kw >= 4;
}


// plan_conv_tc context: the op runs alone (singleton stage / t(v) profiling)
// or next to other ops of its stage
static thread_local bool g_conv_solo = false;
// SM count of the device whose closures are being built (plan_conv_tc)
static thread_local int g_num_sms = 148;
// build_op of a plain tcgen05 conv records its launch descriptor here (the
// group-context build only), so a stage's convs can share one launch
static thread_local std::vector<ConvTcOp>* g_tc_out = nullptr;
static thread_local size_t* g_tc_smem = nullptr;
// where conv_closure<bf16> records its tile plan (OpExec::plan / plan_solo)
static thread_local int* g_plan_out = nullptr;

void ck(cudaError_t e, const char* what) {
  if (e != cudaSuccess) fail(HIOS_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

static inline int rup(int x, int m) { return (x + m - 1) / m * m; }
static inline int64_t rup64(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

Executor::Executor(Schedule& sch) : s(sch), g(*sch.g), M(sch.M) {
  esz = g.dtype == HIOS_BF16 ? 2 : 4;
  group_convs = sch.stage_mode == HIOS_STAGE_GROUPED;
  dataflow = sch.stage_mode == HIOS_STAGE_DATAFLOW;
  auto_pending = sch.stage_mode == HIOS_STAGE_AUTO;
  mode_used = auto_pending ? HIOS_STAGE_STREAMS : sch.stage_mode;
  transport = sch.transport;
  int ndev = 0;
  ck(cudaGetDeviceCount(&ndev), "cudaGetDeviceCount");
  if (ndev <= 0) fail(HIOS_E_CUDA, "no CUDA device");
  lg.resize(M);
  for (int i = 0; i < M; ++i) {
    lg[i].dev = s.devices.empty() ? i % ndev : s.devices[i];
    if (lg[i].dev < 0 || lg[i].dev >= ndev) fail(HIOS_E_INVALID, "device out of range");
    lg[i].local = s.owner.empty() || s.owner[i] == s.rank;
  }
  n_streams = 1;
  for (auto& q : s.Q)
    for (auto& S : q) n_streams = std::max(n_streams, (int)S.size());
}

Executor::~Executor() {
  for (int i = 0; i < M; ++i) {
    LGpu& L = lg[i];
    if (!L.local && !L.ipc_mapped) continue;
    cudaSetDevice(L.dev);
    if (L.ipc_mapped) {
      if (L.arena) cudaIpcCloseMemHandle(L.arena);
      if (L.sync) cudaIpcCloseMemHandle(L.sync);
      continue;
    }
    if (L.gexec) cudaGraphExecDestroy(L.gexec);
    if (L.gexec_timed) cudaGraphExecDestroy(L.gexec_timed);
    if (L.gexec_alt) cudaGraphExecDestroy(L.gexec_alt);
    if (L.gexec_timed_alt) cudaGraphExecDestroy(L.gexec_timed_alt);
    for (auto st : L.streams) cudaStreamDestroy(st);
    if (L.ev_fork) cudaEventDestroy(L.ev_fork);
    for (auto e : L.ev_join) cudaEventDestroy(e);
    if (L.ev_start) cudaEventDestroy(L.ev_start);
    if (L.ev_done) cudaEventDestroy(L.ev_done);
    if (L.arena) cudaFree(L.arena);
    if (L.sync) cudaFree(L.sync);
    for (void* p : L.allocs) cudaFree(p);
  }
  for (auto& x : xfers) {
    if (x.ev_ready) cudaEventDestroy(x.ev_ready);
    if (x.ev_recv) cudaEventDestroy(x.ev_recv);
  }
  for (auto& kv : edge_ev) cudaEventDestroy(kv.second);
  for (auto& L : lg)
    if (L.comm) cudaStreamDestroy(L.comm);
  nccl_comm_destroy(comm);
  for (auto e : op_ev0) if (e) cudaEventDestroy(e);
  for (auto e : op_ev1) if (e) cudaEventDestroy(e);
  if (d_in_stage) cudaFree(d_in_stage);
  if (d_out_stage) cudaFree(d_out_stage);
}

// ----------------------------------------------------------------- plan
void Executor::plan() {
  const int n = g.n;
  std::vector<std::vector<char>> need(n, std::vector<char>(M, 0));
  for (int u = 0; u < n; ++u) {
    need[u][s.gpu_of[u]] = 1;
    for (int e : g.ops[u].out_edges) need[u][s.gpu_of[g.edges[e].dst]] = 1;
  }
  loc.assign(n, std::vector<Loc>(M));
  inplace.assign(g.edges.size(), 0);
  std::vector<int64_t> cursor(M, 0);
  auto alloc = [&](int l, int64_t bytes) {
    int64_t off = cursor[l];
    // +128 B of (zeroed) slack: a conv whose C is not a multiple of 64 reads
    // its last chunk as overlapping 64-channel windows (see conv_closure)
    cursor[l] += rup64(std::max<int64_t>(bytes, 16) + 128, 256);
    return off;
  };
  // ReLU hoisting (relu_out): an op whose every consumer applies ReLU to it
  // first stores its output ReLU'd (its epilogue has a ReLU flag: conv,
  // separable conv, add, identity).  A concat whose consumers all do is stored
  // ReLU'd: each input that qualifies (the concat counted as ReLU-first) writes
  // its slice ReLU'd in place; any other input keeps its raw output in its own
  // buffer and the concat ReLU-copies that slice (relu_copy_in) -- NASNet's
  // cell outputs: the five branch adds in place, the fitted input copied
  relu_out.assign(n, 0);
  relu_copy_in.assign(g.edges.size(), 0);
  {
    auto relu_first = [&](int v) {
      const Op& c = g.ops[v];
      // (a separable conv aggregates its inputs before the ReLU: one input only)
      const bool single = c.in_edges.size() == 1 && (c.agg.empty() || c.agg[0] == 1.f);
      if (c.kind == HIOS_OP_CONV && c.pre_relu) return true;
      if (c.kind == HIOS_OP_SEPCONV && c.pre_relu && single) return true;
      return c.kind == HIOS_OP_ADD && c.relu && single;
    };
    auto can_relu = [&](int u) {
      const int k = g.ops[u].kind;
      return u != g.sink_op && (k == HIOS_OP_CONV || k == HIOS_OP_SEPCONV || k == HIOS_OP_ADD || k == HIOS_OP_IDENTITY);
    };
    auto all_relu_first = [&](int u, int except) {
      if (g.ops[u].out_edges.empty()) return false;
      for (int e : g.ops[u].out_edges) {
        const int v = g.edges[e].dst;
        if (v != except && !relu_first(v)) return false;
      }
      return true;
    };
    for (int c = 0; c < n; ++c) {
      if (g.ops[c].kind != HIOS_OP_CONCAT || c == g.sink_op || !all_relu_first(c, -1)) continue;
      relu_out[c] = 1;
      for (int e : g.ops[c].in_edges) {
        const int p = g.edges[e].src;
        bool ok = can_relu(p) && all_relu_first(p, c);
        for (int e2 : g.ops[p].out_edges)  // a producer of two concats: copy
          if (g.edges[e2].dst != c && g.ops[g.edges[e2].dst].kind == HIOS_OP_CONCAT) ok = false;
        if (ok) relu_out[p] = 1;
        else relu_copy_in[e] = 1;
      }
    }
    for (int u = 0; u < n; ++u)
      if (!relu_out[u] && can_relu(u) && all_relu_first(u, -1)) relu_out[u] = 1;
  }
  // reverse topological order: a concat consumer's buffer exists before its producers are placed
  for (int k = n - 1; k >= 0; --k) {
    const int u = g.topo[k];
    const Op& o = g.ops[u];
    for (int l = 0; l < M; ++l) {
      if (!need[u][l]) continue;
      bool placed = false;
      for (int e : o.out_edges) {
        const int v = g.edges[e].dst;
        const Op& ov = g.ops[v];
        if (ov.kind != HIOS_OP_CONCAT || s.gpu_of[v] != l || loc[v][l].off < 0 || relu_copy_in[e]) continue;
        int c_off = 0;
        for (int e2 : ov.in_edges) {
          if (g.edges[e2].slot >= g.edges[e].slot) break;
          c_off += g.ops[g.edges[e2].src].C;
        }
        if (c_off % 8 || loc[v][l].ldc % 8) continue;  // 16-byte aligned slices only
        loc[u][l] = Loc{loc[v][l].off + (int64_t)c_off * esz, loc[v][l].ldc};
        inplace[e] = 1;
        placed = true;
        break;
      }
      if (!placed) {
        const int ldc = rup(o.C, 8);
        loc[u][l] = Loc{alloc(l, (int64_t)o.H * o.W * ldc * esz), ldc};
      }
    }
  }
  ox.assign(n, OpExec());
  for (int v = 0; v < n; ++v) {
    const Op& o = g.ops[v];
    const int l = s.gpu_of[v];
    if (o.kind == HIOS_OP_CONV && g.dtype == HIOS_BF16 && s2d_conv(o)) {
      OpExec& x = ox[v];
      x.s2d_ldc = rup(4 * o.in_c, 8);
      x.s2dbuf = alloc(l, ((int64_t)(o.H + (o.kh + 1) / 2 - 1) * (o.W + (o.kw + 1) / 2 - 1) + 4) * x.s2d_ldc * esz);
    }
    if (o.kind == HIOS_OP_SEPCONV) {
      OpExec& x = ox[v];
      x.dw_ldc = rup(std::max(o.in_c, o.out_c), 8);
      x.dwbuf = alloc(l, (int64_t)o.H * o.W * x.dw_ldc * esz);
      if (o.reps > 1) {
        x.mid_ldc = rup(o.out_c, 8);
        x.midbuf = alloc(l, (int64_t)o.H * o.W * x.mid_ldc * esz);
      }
    }
  }
  // pre-ReLU convs: one ReLU'd copy of the input per (producer, GPU) when the
  // producer runs on that GPU (made right after it), else a per-consumer scratch
  relu_loc.clear();
  for (int v = 0; v < n; ++v) {
    const Op& o = g.ops[v];
    if (o.kind != HIOS_OP_CONV || !o.pre_relu) continue;
    if (relu_out[g.edges[o.in_edges[0]].src]) continue;  // stored ReLU'd already
    const int u = g.edges[o.in_edges[0]].src, l = s.gpu_of[v];
    const Op& ou = g.ops[u];
    const int ldc = rup(ou.C, 8);
    const int64_t bytes = (int64_t)ou.H * ou.W * ldc * esz;
    if (s.gpu_of[u] == l && ou.kind != HIOS_OP_INPUT) {
      const int64_t key = (int64_t)u * M + l;
      if (!relu_loc.count(key)) relu_loc[key] = Loc{alloc(l, bytes), ldc};
    } else {
      ox[v].relubuf = alloc(l, bytes);
      ox[v].relu_ldc = ldc;
    }
  }
  // remote deliveries and flags
  flag_index.assign(n, std::vector<int>(M, -1));
  std::vector<int> nflags(M, 0);
  for (int u = 0; u < n; ++u) {
    const int home = s.gpu_of[u];
    const int kind = g.ops[u].kind;
    const bool can_fuse = kind == HIOS_OP_CONV || kind == HIOS_OP_SEPCONV || kind == HIOS_OP_MAXPOOL ||
                          kind == HIOS_OP_AVGPOOL || kind == HIOS_OP_ADD;
    for (int l = 0; l < M; ++l) {
      if (l == home || !need[u][l]) continue;
      const bool cross_proc = !s.owner.empty() && s.owner[l] != s.owner[home];
      int mode;
      if (transport == HIOS_TRANSPORT_NCCL && cross_proc) mode = DM_NCCL;
      else if (transport == HIOS_TRANSPORT_PEER) mode = can_fuse ? DM_FUSED : DM_PUSH;
      else mode = DM_COPY;  // copy transport; NCCL between logical GPUs of one process
      if (mode != DM_NCCL) flag_index[u][l] = nflags[l]++;
      ox[u].remote.push_back({l, mode});
    }
  }
  // NCCL transfers in the global order; a transfer whose two buffers are not
  // both whole [H*W][ldc] tensors with the same pitch goes through packed
  // [H*W][C] staging buffers on both sides
  xfers.clear();
  if (transport == HIOS_TRANSPORT_NCCL) {
    for (auto& pr : transfer_order(s)) {
      const int u = pr.first, d = pr.second;
      bool nc = false;
      for (auto& r : ox[u].remote)
        if (r.gpu == d && r.mode == DM_NCCL) nc = true;
      if (!nc) continue;
      const Op& o = g.ops[u];
      NcclXfer x;
      x.u = u;
      x.src = s.gpu_of[u];
      x.dst = d;
      const int lw = rup(o.C, 8);
      if (loc[u][x.src].ldc == lw && loc[u][d].ldc == lw) {
        x.bytes = (size_t)o.H * o.W * lw * esz;
      } else {
        x.bytes = (size_t)o.H * o.W * o.C * esz;
        x.send_off = alloc(x.src, (int64_t)x.bytes);
        x.recv_off = alloc(d, (int64_t)x.bytes);
      }
      xfers.push_back(x);
    }
  }
  for (int l = 0; l < M; ++l) {
    lg[l].arena_bytes = (size_t)std::max<int64_t>(cursor[l], 256);
    lg[l].sync_words = 1 + M + nflags[l];
  }
}

// ------------------------------------------------------------- allocate
template <typename T> static T to_dev_t(float x);
template <> float to_dev_t<float>(float x) { return x; }
template <> bf16 to_dev_t<bf16>(float x) { return __float2bfloat16(x); }

template <typename T>
static void* upload(LGpu& L, const std::vector<T>& h) {
  void* d = nullptr;
  ck(cudaMalloc(&d, std::max<size_t>(h.size() * sizeof(T), 16)), "cudaMalloc weights");
  L.allocs.push_back(d);
  if (!h.empty()) ck(cudaMemcpy(d, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice), "upload");
  return d;
}

// conv weights W[k][c][r][s] -> tensor-core layout [k][r*S+s][Cp] (Cp = C rounded to 8, zero pad)
//                             -> SIMT layout [k][r][s][c]
// fold (tcgen05 convs): the folded-BN scale of output channel k is multiplied
// into its weights before rounding to bf16 (scale * (W * x) = (scale W) * x),
// so the conv_tc epilogue adds the shift only
template <typename T>
static std::vector<T> conv_layout(const float* W, int K, int C, int R, int S, int Cp, const float* fold = nullptr) {
  std::vector<T> out((size_t)K * R * S * Cp, to_dev_t<T>(0.f));
  for (int k = 0; k < K; ++k) {
    const float f = fold ? fold[k] : 1.f;
    for (int c = 0; c < C; ++c)
      for (int r = 0; r < R; ++r)
        for (int s2 = 0; s2 < S; ++s2)
          out[((size_t)k * R * S + r * S + s2) * Cp + c] = to_dev_t<T>(f * W[(((size_t)k * C + c) * R + r) * S + s2]);
  }
  return out;
}

// stems (C <= 8, receptive field <= 49 taps, weights fit in smem): direct CUDA-core kernel
// (the fp32 path; the bf16 path takes s2d_conv first)
static bool small_c_conv(const Op& o) {
  return o.in_c <= 8 && o.kh * o.kw <= 49 && (size_t)o.out_c * o.kh * o.kw * o.in_c * 4 <= 96 * 1024 && o.dh == 1 &&
         o.dw == 1;
}

template <typename T>
static void upload_weights_T(Executor& ex, int v) {
  const Op& o = ex.g.ops[v];
  LGpu& L = ex.lg[ex.s.gpu_of[v]];
  OpExec& x = ex.ox[v];
  const bool tc = ex.g.dtype == HIOS_BF16;
  switch (o.kind) {
    case HIOS_OP_CONV: {
      // bf16: whole 64-channel chunks, fp32 SIMT: whole 16-channel chunks (zero-padded)
      const int Cp = tc ? rup(o.in_c, 64) : rup(o.in_c, 16);
      if (tc && s2d_conv(o)) {
        // W'[k][r'*S'+s'][(a*2+b)*C + c] (see s2d_conv)
        const int R2 = (o.kh + 1) / 2, S2 = (o.kw + 1) / 2, C = o.in_c, Cp2 = rup(4 * C, 64);
        std::vector<T> w2((size_t)o.out_c * R2 * S2 * Cp2, to_dev_t<T>(0.f));
        for (int k = 0; k < o.out_c; ++k)
          for (int c = 0; c < C; ++c)
            for (int r = 0; r < o.kh; ++r)
              for (int s2 = 0; s2 < o.kw; ++s2) {
                const int ch = ((r & 1) * 2 + (s2 & 1)) * C + c;
                w2[((size_t)k * R2 * S2 + (r >> 1) * S2 + (s2 >> 1)) * Cp2 + ch] =
                    to_dev_t<T>(o.scale[k] * o.weight[(((size_t)k * C + c) * o.kh + r) * o.kw + s2]);
              }
        x.w = upload(L, w2);
        if (rup(4 * C, 8) == 16 && S2 <= 4) {
          // packed taps: one 64-element K row per r' = S2 taps x 16 channels
          // (zero weights for the taps s' >= S2 the 4-pixel window also covers)
          std::vector<T> w3((size_t)o.out_c * R2 * 64, to_dev_t<T>(0.f));
          for (int k = 0; k < o.out_c; ++k)
            for (int r2 = 0; r2 < R2; ++r2)
              for (int s2 = 0; s2 < S2; ++s2)
                for (int ch = 0; ch < 16; ++ch)
                  w3[((size_t)k * R2 + r2) * 64 + s2 * 16 + ch] = w2[((size_t)k * R2 * S2 + r2 * S2 + s2) * Cp2 + ch];
          x.w_pack = upload(L, w3);
        }
        x.scale.push_back((float*)upload(L, o.scale));
        x.shift.push_back((float*)upload(L, o.shift));
        break;
      }
      if (!small_c_conv(o) && o.kh * o.kw > 1 && !o.weight.empty()) {
        // single non-zero tap: keep only that tap (x.tap_r / tap_s)
        int nz = 0, r0 = -1, s0 = -1;
        for (int r = 0; r < o.kh && nz < 2; ++r)
          for (int s2 = 0; s2 < o.kw && nz < 2; ++s2) {
            bool any = false;
            for (int k = 0; k < o.out_c && !any; ++k)
              for (int c = 0; c < o.in_c; ++c)
                if (o.weight[(((size_t)k * o.in_c + c) * o.kh + r) * o.kw + s2] != 0.f) { any = true; break; }
            if (any) { ++nz; r0 = r; s0 = s2; }
          }
        if (nz == 1) {
          std::vector<float> w1((size_t)o.out_c * o.in_c);
          for (int k = 0; k < o.out_c; ++k)
            for (int c = 0; c < o.in_c; ++c)
              w1[(size_t)k * o.in_c + c] = o.weight[(((size_t)k * o.in_c + c) * o.kh + r0) * o.kw + s0];
          x.w = upload(L, conv_layout<T>(w1.data(), o.out_c, o.in_c, 1, 1, Cp, tc ? o.scale.data() : nullptr));
          x.tap_r = r0;
          x.tap_s = s0;
          x.scale.push_back((float*)upload(L, o.scale));
          x.shift.push_back((float*)upload(L, o.shift));
          break;
        }
      }
      x.w = upload(L, conv_layout<T>(o.weight.data(), o.out_c, o.in_c, o.kh, o.kw, Cp, tc ? o.scale.data() : nullptr));
      if (small_c_conv(o)) x.w_small = (float*)upload(L, conv_layout<float>(o.weight.data(), o.out_c, o.in_c, o.kh, o.kw, o.in_c));
      x.scale.push_back((float*)upload(L, o.scale));
      x.shift.push_back((float*)upload(L, o.shift));
      break;
    }
    case HIOS_OP_SEPCONV: {
      size_t off = 0;
      for (int r = 0; r < o.reps; ++r) {
        const int c = r == 0 ? o.in_c : o.out_c;
        const int RS = o.kh * o.kw;
        std::vector<float> dw((size_t)RS * c);
        for (int ch = 0; ch < c; ++ch)
          for (int rs = 0; rs < RS; ++rs) dw[(size_t)rs * c + ch] = o.weight[off + (size_t)ch * RS + rs];
        off += (size_t)c * RS;
        x.dw.push_back((float*)upload(L, dw));
        const int Cp = tc ? rup(c, 64) : rup(c, 16);
        x.pw.push_back(upload(L, conv_layout<T>(o.weight.data() + off, o.out_c, c, 1, 1, Cp,
                                                tc ? o.scale.data() + (size_t)r * o.out_c : nullptr)));
        off += (size_t)o.out_c * c;
        std::vector<float> sc(o.scale.begin() + (size_t)r * o.out_c, o.scale.begin() + (size_t)(r + 1) * o.out_c);
        std::vector<float> sh(o.shift.begin() + (size_t)r * o.out_c, o.shift.begin() + (size_t)(r + 1) * o.out_c);
        x.scale.push_back((float*)upload(L, sc));
        x.shift.push_back((float*)upload(L, sh));
      }
      break;
    }
    case HIOS_OP_LINEAR: {
      // weight columns follow the NCHW flatten order; the input is NHWC:
      // only C x 1 x 1 inputs (flatten orders coincide) are supported
      const int in_op = ex.g.edges[o.in_edges[0]].src;
      const Op& xi = ex.g.ops[in_op];
      if (xi.H * xi.W != 1) fail(HIOS_E_UNSUPPORTED, "linear on a spatial input (insert a GAP)");
      x.ldw = rup(o.in_c, 8);
      std::vector<T> w((size_t)o.out_c * x.ldw, to_dev_t<T>(0.f));
      for (int k = 0; k < o.out_c; ++k)
        for (int c = 0; c < o.in_c; ++c) w[(size_t)k * x.ldw + c] = to_dev_t<T>(o.weight[(size_t)k * o.in_c + c]);
      x.w = upload(L, w);
      x.bias = (float*)upload(L, o.shift);
      break;
    }
    default:
      break;
  }
}

void Executor::allocate() {
  // peer access between distinct local devices
  std::set<int> devs;
  for (auto& L : lg) if (L.local) devs.insert(L.dev);
  for (int a : devs)
    for (int b : devs) {
      if (a == b) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, a, b);
      if (can) {
        cudaSetDevice(a);
        cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
          ck(e, "cudaDeviceEnablePeerAccess");
        cudaGetLastError();
      }
    }
  for (int l = 0; l < M; ++l) {
    LGpu& L = lg[l];
    if (!L.local) continue;
    ck(cudaSetDevice(L.dev), "cudaSetDevice");
    ck(cudaMalloc(&L.arena, L.arena_bytes), "cudaMalloc arena");
    ck(cudaMemset(L.arena, 0, L.arena_bytes), "memset arena");
    ck(cudaMalloc(&L.sync, L.sync_words * sizeof(unsigned)), "cudaMalloc sync");
    ck(cudaMemset(L.sync, 0, L.sync_words * sizeof(unsigned)), "memset sync");
    L.streams.resize(n_streams);
    for (auto& st : L.streams) ck(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking), "stream");
    ck(cudaEventCreateWithFlags(&L.ev_fork, cudaEventDisableTiming), "event");
    L.ev_join.resize(n_streams);
    for (auto& e : L.ev_join) ck(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event");
    ck(cudaEventCreate(&L.ev_start), "event");
    ck(cudaEventCreate(&L.ev_done), "event");
    ck(cudaDeviceGetAttribute(&L.num_sms, cudaDevAttrMultiProcessorCount, L.dev), "SM count");
  }
  // one CUDA graph per device (its local logical GPUs), owner = the first
  graphs_by_dev.clear();
  graph_of.assign(M, -1);
  for (int l = 0; l < M; ++l)
    if (lg[l].local) graphs_by_dev[lg[l].dev].push_back(l);
  for (auto& kv : graphs_by_dev)
    for (int l : kv.second) graph_of[l] = kv.second[0];
  for (int u = 0; u < g.n; ++u)
    for (auto& r : ox[u].remote)
      if (same_graph(s.gpu_of[u], r.gpu)) {
        ck(cudaSetDevice(lg[r.gpu].dev), "cudaSetDevice");
        cudaEvent_t e;
        ck(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event");
        edge_ev[(int64_t)u * M + r.gpu] = e;
      }
  for (auto& x : xfers) {
    for (int side = 0; side < 2; ++side) {
      const int l = side ? x.dst : x.src;
      if (!lg[l].local) continue;
      ck(cudaSetDevice(lg[l].dev), "cudaSetDevice");
      LGpu& Lo = lg[graph_of[l]];
      if (!Lo.comm) ck(cudaStreamCreateWithFlags(&Lo.comm, cudaStreamNonBlocking), "comm stream");
      cudaEvent_t& e = side ? x.ev_recv : x.ev_ready;
      ck(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event");
    }
  }
  if (!xfers.empty() && !comm)
    fail(HIOS_E_STATE, "NCCL transport: call hios_schedule_nccl_init before the first run");
  for (int v = 0; v < g.n; ++v) {
    const int l = s.gpu_of[v];
    if (!lg[l].local) continue;
    ck(cudaSetDevice(lg[l].dev), "cudaSetDevice");
    if (g.dtype == HIOS_BF16) upload_weights_T<bf16>(*this, v);
    else upload_weights_T<float>(*this, v);
  }
  lowered = true;
}

// --------------------------------------------------------------- closures
// Tile plan of one tcgen05 conv (see conv_tc.cu): halo mode for stride-1-in-W
// convs with wide outputs, tap mode otherwise; n_tile from a small cost model
// (waves x per-K-step time, where a K-step costs max(MMA, L2->SM bytes)).
static ConvTcArgs plan_conv_tc(int P, int Q, int K, int C, int R, int S, int sh, int sw, int dh, int dw,
                               bool allow_hk = true) {
  ConvTcArgs c{};
  c.hk = 1;
  int hw = 128 + (S - 1) * dw;
  c.halo = (sw == 1 && Q >= 96 && hw <= 256 && R * dh <= 256 && halo_bytes_of(R, hw) <= 100 * 1024) ? 1 : 0;
  // virtual-grid halo (narrow stride-1 square convs, see ConvTcArgs): tap
  // mode would stream the input R*S times through L2->SM; the box of whole
  // padded rows streams it ~(128 + (R-1) dh Wh + (S-1) dw) / 128 times.
  // Measured (tools/op_times.py, Inception-1024): 3x3 at 30^2 15.6 -> 13.5 us,
  // but 7x1 at 62^2 8.8 -> 9.9 us (a 10-row box per 128 outputs) and 1x3 /
  // 3x1 at 30^2 +1 us: square kernels only
  const int Wh = Q + (S - 1) * dw;
  const int vrows = (Wh - 1 + 127 + (S - 1) * dw) / Wh + 1 + (R - 1) * dh;
  static const bool novgrid = getenv("HIOS_NOVGRID") != nullptr;  // A/B switch
  if (!c.halo && !novgrid && sh == 1 && sw == 1 && dh == 1 && dw == 1 && R == S && R >= 3 && Wh <= 256 && vrows <= 256 &&
      halo_bytes_of(vrows, Wh) <= 96 * 1024) {
    c.halo = 1;
    c.vgrid = Wh;
    hw = Wh;
  }
  if (c.halo) {
    c.th = 1;
    c.tw = 128;
    c.halo_w = hw;
    c.hrows = c.vgrid ? vrows : R;
    c.hrow_px = c.vgrid ? dh * Wh : hw;
  } else {
    int64_t best = -1;
    for (int tw : {128, 64, 32, 16, 8}) {
      const int th = 128 / tw;
      if (tw * sw > 256 || th * sh > 256) continue;
      const int64_t cost = (int64_t)((P + th - 1) / th) * th * ((Q + tw - 1) / tw) * tw;
      if (best < 0 || cost < best) { best = cost; c.th = th; c.tw = tw; }
    }
    if (best < 0) fail(HIOS_E_UNSUPPORTED, "conv stride too large for the TMA box");
  }
  // row groups (classic halo, stride 1, shapes with an unrolled tap loop):
  // two output rows per tile share one box of R + 1 input rows and every
  // weight stage (B) -- per output row, R -> (R + 1) / 2 input rows and half
  // the weight bytes cross L2 -> SM (the halo convs at 2048^2 / 4096^2 are
  // bound by the TMA's per-row processing, profiles/README.md)
  static const bool nohk = getenv("HIOS_NOHK") != nullptr;  // A/B switch
  const bool hk_shape = (R == 3 && S == 3) || (R == 5 && S == 5) || (R == 7 && S == 1) || (R == 3 && S == 1) ||
                        (R == 2 && S == 1) || (R == 4 && S == 1);
  if (allow_hk && !nohk && c.halo && !c.vgrid && sh == 1 && dh == 1 && hk_shape && P >= 4) {
    c.hk = 2;
    c.th = 2;
    c.hrows = R + 1;
  }
  // pixel pairs (1x1, stride 1, wide rows): a tile is 256 consecutive pixels of
  // one output row as two 128-pixel accumulators sharing every weight stage
  // (one box of 256 pixels per channel chunk): half the weight bytes per output
  if (allow_hk && !nohk && c.halo && !c.vgrid && R == 1 && S == 1 && sh == 1 && Q >= 192) {
    c.hk = 2;
    c.hk_px = 1;
    c.tw = 256;
    c.halo_w = 256;
    hw = 256;
    c.hrow_px = 128;  // accumulator j reads the window j * 128 pixels into the box
  }
  c.tiles_q = (Q + c.tw - 1) / c.tw;
  c.tiles_m = ((P + c.th - 1) / c.th) * c.tiles_q;
  if (c.vgrid) {
    c.tiles_q = 1;
    c.tiles_m = (int)(((int64_t)P * c.vgrid + 127) / 128);
  }
  c.c_chunks = (C + 63) / 64;
  const int KI = R * S * c.c_chunks;
  // cost model (cycles), from the measured issue costs on B200
  // (tools/mma_bench.cu, tools/tma_bench.cu): ~100 cycles per tcgen05.mma and
  // ~500 per TMA instruction per issuing thread; MMA M=128 x N x K=16 takes
  // N/2 cycles; ~64 B/cycle/SM of TMA bandwidth.
  auto n_mma_of = [](int nt) { return nt % 64 == 0 ? 4 : (nt % 32 == 0 ? 2 : 1); };
  double best_cost = 1e300;
  for (int nt = 16; nt <= 256; nt += 16) {
    if (nt > rup(K, 16)) break;
    const int tn = (K + nt - 1) / nt;
    const int nm = n_mma_of(nt);
    const double mma = std::max(4.0 * nt / 2.0, 4.0 * 100.0 / nm);
    const double a_bytes = c.halo ? (double)c.hrows * c.halo_w * 128.0 / (R * S) : 16384.0;
    const double tma = std::max((c.halo ? 1.0 : 2.0) * 500.0 / 4.0, (a_bytes + nt * 128.0) / 64.0);
    const double epi = nt / 16.0 * 80.0 + 128.0 * nt * 2.0 / 64.0;
    const double tile = std::max(KI * std::max(mma, tma), epi) + 300.0;
    const double waves = std::ceil((double)c.tiles_m * tn / (double)g_num_sms);
    const double cost = waves * tile + 1500.0;
    if (cost < best_cost * 0.98) { best_cost = cost; c.n_tile = nt; }
  }
  if (c.vgrid && !g_conv_solo) {
    // virtual-grid halo next to other ops of its stage: the tap-mode rule
    // (widest N tile <= 128 that splits K evenly) -- fewer CTAs, since the
    // stage's concurrent ops already fill the SMs (measured: the cost model's
    // 64-wide tiles made Inception-1024 HIOS-LP 0.74 -> 0.84 ms)
    const int nb = (K + 127) / 128;
    c.n_tile = rup((K + nb - 1) / nb, 16);
  }
  if (!c.halo) {
    // tap mode: the per-stage cost is dominated by a fixed handshake
    // (measured), so take a wide N tile (<= 128) that splits K evenly
    // (measured: halving helps ops run alone but loses under HIOS stages,
    // where concurrent ops already fill the SMs -- kept as HIOS_TAPCAP)
    // alone on the GPU (singleton stage) a 64-wide tile doubles the CTAs
    // (measured: sequential Inception-1024 1.077 -> 0.981 ms with 64 for all)
    // (only when 128-wide tiles leave SMs idle)
    int cap = (g_conv_solo && (int64_t)c.tiles_m * ((K + 127) / 128) < g_num_sms) ? 64 : 128;
    const int nb = (K + cap - 1) / cap;
    c.n_tile = rup((K + nb - 1) / nb, 16);
  }
  c.tiles_n = (K + c.n_tile - 1) / c.n_tile;
  // row groups need 2 * hk * n_tile <= 512 TMEM columns and pay only with
  // enough tiles to fill the SMs twice (measured, tools/conv_micro.py: forcing
  // n_tile <= 128 made Mixed_7b 3x3 at 126^2 49.7 -> 59.4 us; halving the tiles
  // of Conv2d_4a at 254^2 29.6 -> 31.8 us; 2a / 2b / 5x5 at 4096^2 -16..-23 %)
  // (measured: with n_tile 192 and one accumulator set -- no epilogue overlap
  // -- Conv2d_4a at 4096^2 371 -> 379 us, so row groups keep two sets)
  if (c.hk > 1 && (c.n_tile > 128 || (int64_t)c.tiles_m * c.tiles_n < 2LL * g_num_sms))
    return plan_conv_tc(P, Q, K, C, R, S, sh, sw, dh, dw, false);
  // TMEM accumulator sets of hk x n_tile columns (the kernel supports 1 when
  // 2 sets do not fit in 512 columns)
  c.nacc = 2 * c.hk * c.n_tile <= 512 ? 2 : 1;
  c.n_mma = 1;  // measured: splitting N over several MMA warps does not pay (tools/conv_micro.py)
  const size_t B = (size_t)c.n_tile * 128;
  const size_t stage_out = 128 * ((size_t)c.n_tile * 2 + 16);
  // epilogue: two staging tiles for N tiles <= 128 (the stores of tile i
  // drain while tile i+1 is staged), folded BN resident when K is small
  // one CTA per SM: 164 registers x 384 threads (the kernel also takes the
  // whole TMEM on that basis)
  c.occ = 1;
  // epilogue mode (HIOS_EPI overrides): direct register stores for N tiles
  // <= 128 (no staging tile), TMA bulk-tensor stores for wider tiles
  c.epi = (c.n_tile <= 128 || c.hk > 1) ? 2 : 1;  // row groups: direct stores (any n_tile)
  c.out_bufs = c.epi == 2 ? 0 : (c.n_tile <= (c.occ == 2 ? 48 : 128) ? 2 : 1);
  c.sres = c.tiles_n * c.n_tile <= kScaleRes ? 1 : 0;
  // occupancy: 1 CTA/SM (212 KB) or 2 CTAs/SM (104 KB each, TMEM <= 256 cols)
  const size_t budget = (c.occ == 2 ? 104 * 1024 : 212 * 1024) - c.out_bufs * stage_out;
  // K-steps per stage: amortise the ~0.3 us full/empty handshake (measured)
  c.kps = 0;
  // resident weights (halo mode, one N tile, CTAs that walk several tiles):
  // the whole B is loaded once per CTA instead of once per tile (measured:
  // Conv2d_2a re-read 36 KB of weights per 25 KB input tile)
  const size_t b_all = (size_t)c.c_chunks * R * S * B;
  c.bres = 0;
  if (c.halo && c.tiles_n == 1 && c.tiles_m > g_num_sms * c.occ && b_all <= 96 * 1024 &&
      halo_bytes_of(c.hrows, hw) + b_all <= budget) {
    c.bres = 1;
    c.kps = std::min(4, R * S);
    // as many input boxes in flight as fit (measured: the halo TMA latency,
    // ~2 us, bounds a 2-deep ring at small K; tools/conv_trace2.py)
    const int cap = kMaxABufs;
    c.a_bufs = 1;
    while (c.a_bufs < cap && (c.a_bufs + 1) * halo_bytes_of(c.hrows, hw) + b_all <= budget) ++c.a_bufs;
    c.stages = 2;
  }
  if (c.halo && !c.bres) {
    const size_t H = halo_bytes_of(c.hrows, hw);
    if (!c.kps) c.kps = std::min(4, R * S);
    while (c.kps > 1 && H + 2 * c.kps * B > budget) --c.kps;
    c.a_bufs = (2 * H + 2 * c.kps * B <= budget) ? 2 : 1;
    {  // deeper input ring while >= 4 B stages still fit
      const int cap = 4;
      while (c.a_bufs < cap && (c.a_bufs + 1) * H + 4 * c.kps * B <= budget) ++c.a_bufs;
    }
    if (H + 2 * c.kps * B > budget) {
      if (c.hk > 1) return plan_conv_tc(P, Q, K, C, R, S, sh, sw, dh, dw, false);
      fail(HIOS_E_UNSUPPORTED, "conv halo plan does not fit shared memory");
    }
    else c.stages = (int)std::min<size_t>(8, (budget - c.a_bufs * H) / (c.kps * B));
  }
  if (!c.halo) {
    if (!c.kps) c.kps = 4;
    while (c.kps > 1 && 2 * c.kps * (16384 + B) > budget) --c.kps;
    c.stages = (int)std::min<size_t>(8, budget / (c.kps * (16384 + B)));
  }
  const int n_stage_steps = (KI + c.kps - 1) / c.kps;
  c.stages = std::max(2, std::min(c.stages, std::max(n_stage_steps, 2)));
  // no split-K (measured: a workspace + finalize kernel and a cluster /
  // distributed-shared-memory reduction both lost under HIOS stages,
  // DESIGN.md §6)
  c.ksplit = 1;
  c.kpsplit = KI;
  if (c.hk > 1) {
    // the kernel's row-group loops exist only for the unrolled (R, S, kps)
    // shapes (conv_tc.cu halo_taps_ring / halo_taps_bres) and the direct-store
    // epilogue; anything else plans without row groups
    const bool ring_ok = (R == 3 && S == 3 && c.kps >= 2 && c.kps <= 4) || (R == 5 && S == 5 && c.kps == 4) ||
                         (R == 7 && S == 1 && c.kps == 4) || (R == 3 && S == 1 && c.kps == 3);
    const bool bres_ok = (R == 3 && S == 3) || (R == 2 && S == 1) || (R == 4 && S == 1) || (R == 5 && S == 5) ||
                         (R == 1 && S == 1);
    const bool ring_ok1 = R == 1 && S == 1 && c.kps == 1;
    if (c.epi != 2 || !(c.bres ? bres_ok : (ring_ok || ring_ok1)) || (c.nacc == 1 && c.bres))
      return plan_conv_tc(P, Q, K, C, R, S, sh, sw, dh, dw, false);
  }
  return c;
}

struct View {
  char* p;
  int ldc;
  int row_px = 0;  // pixels per row for the row pitch (0: the conv's W)
};

template <typename T>
static Dst<T> dst_of(const std::vector<View>& v) {
  if ((int)v.size() > kMaxDst) fail(HIOS_E_UNSUPPORTED, "more remote destinations than kMaxDst");
  Dst<T> d{};
  d.n = (int)v.size();
  for (size_t i = 0; i < v.size(); ++i) {
    d.p[i] = (T*)v[i].p;
    d.ld[i] = v[i].ldc;
  }
  return d;
}

template <typename T>
static std::function<void(cudaStream_t)> conv_closure(Executor& ex, const View& in, int H, int W, int C,
                                                      const void* w, float* scale, float* shift, int K, int R,
                                                      int S, int sh, int sw, int ph, int pw, int dh, int dw,
                                                      int P, int Q, int relu, const View& out,
                                                      const std::vector<View>& out2, int& nk);

template <>
std::function<void(cudaStream_t)> conv_closure<bf16>(Executor& ex, const View& in, int H, int W, int C, const void* w,
                                                     float* scale, float* shift, int K, int R, int S, int sh, int sw,
                                                     int ph, int pw, int dh, int dw, int P, int Q, int relu,
                                                     const View& out, const std::vector<View>& out2, int& nk) {
  ConvTcArgs a = plan_conv_tc(P, Q, K, C, R, S, sh, sw, dh, dw);
  CUtensorMap mx, mw;
  bool ok;
  // C % 64 != 0: the tensor map's channel extent is rounded up to whole
  // 64-channel chunks, so the last chunk's box reads past C into the pixel's
  // pad / the next pixel (finite data -- the arena is zeroed and every buffer
  // has 128 B of slack) instead of being zero-filled by TMA: measured
  // (tools/tma_bench.cu) a box with channel out-of-bounds fill streams at
  // ~16 B/cycle/SM whatever the number of issuing warps, 2-7x slower than an
  // in-bounds box.  Those channels meet zero weights (pitch rup(C, 64)) or are
  // skipped (K=16 slices past C are not issued).
  const int Cm = C % 64 ? rup(C, 64) : C;
  if (a.vgrid)  // hrows whole padded input rows (x from -pw) per channel chunk
    ok = make_tmap_3d(&mx, in.p, Cm, W, H, (uint64_t)in.ldc * 2, (uint64_t)(in.row_px ? in.row_px : W) * in.ldc * 2, 64, a.halo_w,
                      a.hrows, 1, 1);
  else if (a.halo)  // R input rows (stride dh) x halo_w pixels per channel chunk
    ok = make_tmap_3d(&mx, in.p, Cm, W, H, (uint64_t)in.ldc * 2, (uint64_t)(in.row_px ? in.row_px : W) * in.ldc * 2, 64, a.halo_w,
                      a.hrows * dh, 1, dh);
  else         // th x tw output positions of one (r, s) tap, conv stride as traversal stride
    ok = make_tmap_3d(&mx, in.p, Cm, W, H, (uint64_t)in.ldc * 2, (uint64_t)(in.row_px ? in.row_px : W) * in.ldc * 2, 64, a.tw * sw, a.th * sh,
                      sw, sh);
  if (!ok) fail(HIOS_E_CUDA, "tensor map (activation)");
  const int Cp = rup(C, 64);  // weight pitch: whole zero-padded 64-channel chunks (no TMA OOB fill)
  if (!make_tmap_3d(&mw, w, Cp, R * S, K, (uint64_t)Cp * 2, (uint64_t)R * S * Cp * 2, 64, 1, a.n_tile, 1, 1))
    fail(HIOS_E_CUDA, "tensor map (weights)");
  a.P = P; a.Q = Q; a.K = K; a.C = C; a.R = R; a.S = S; a.sh = sh; a.sw = sw; a.ph = ph; a.pw = pw;
  a.dh = dh; a.dw = dw; a.relu = relu; a.scale = scale; a.shift = shift;
  a.bo_mode = 0;
  a.trace = getenv("HIOS_TRACE") ? 1 : 0;  // per-CTA globaltimer timeline (tools/conv_trace.py)
  a.spin = 0;
  a.dbg = 0;
  a.out = (bf16*)out.p; a.ldo = out.ldc;
  a.out2 = dst_of<bf16>(out2);
  // 256-bit epilogue stores need every pixel row of every destination
  // 32-byte aligned (16-channel groups of the tile start at n0 % 16 == 0)
  a.st256 = ((uintptr_t)out.p % 32 == 0 && out.ldc % 16 == 0 && !getenv("HIOS_NOST256")) ? 1 : 0;
  for (auto& v : out2)
    if ((uintptr_t)v.p % 32 != 0 || v.ldc % 16 != 0) a.st256 = 0;
  // epilogue by TMA bulk-tensor stores: output tensor map {K, Q, P} over the
  // destination slice (clips the ragged pixel / channel edges of a tile)
  CUtensorMap mo = mx, mo2 = mx;
  a.out_sw = a.n_tile % 64 == 0 ? 64 : (a.n_tile % 32 == 0 ? 32 : 16);
  if (a.vgrid && a.epi == 1) a.epi = 0;  // tiles are not rectangular: no TMA-store boxes
  a.tma_out = a.ksplit == 1 && a.epi == 1 ? 1 : 0;
  if (a.ksplit > 1 || (a.epi == 1 && !a.tma_out)) a.epi = 0;
  if (a.tma_out) {
    const int sb = a.out_sw * 2;
    // one box = one epilogue warp's 32 rows of the 128-pixel tile
    const uint32_t bw = (uint32_t)std::min(a.tw, 32), bh = 32u / bw;
    a.tma_out = make_tmap_3d(&mo, out.p, K, Q, P, (uint64_t)out.ldc * 2, (uint64_t)Q * out.ldc * 2, a.out_sw, bw, bh,
                             1, 1, sb) &&
                (out2.empty() || (out2.size() == 1 && make_tmap_3d(&mo2, out2[0].p, K, Q, P, (uint64_t)out2[0].ldc * 2,
                                                                   (uint64_t)Q * out2[0].ldc * 2, a.out_sw, bw, bh, 1,
                                                                   1, sb)));
    if (!a.tma_out) a.epi = 0;
  }
  const size_t smem = conv_tc_smem_bytes(a);
  if (g_plan_out) {
    const int pl[8] = {a.vgrid ? 3 : (a.halo ? 2 : 1), a.n_tile, a.tiles_m * a.tiles_n, a.epi, a.st256, a.hk,
                       a.stages, a.kps};
    std::memcpy(g_plan_out, pl, sizeof(pl));
  }
  const int grid = std::min(a.tiles_m * a.tiles_n * a.ksplit, g_num_sms * a.occ);
  nk += 1;
  if (g_tc_out) {
    ConvTcOp op;
    op.mx = mx; op.mw = mw; op.mo = mo; op.mo2 = mo2; op.a = a;
    g_tc_out->push_back(op);
    *g_tc_smem = std::max(*g_tc_smem, smem);
  }
  return [mx, mw, mo, mo2, a, smem, grid](cudaStream_t st) { launch_conv_tc(mx, mw, mo, mo2, a, grid, smem, st); };
}

template <>
std::function<void(cudaStream_t)> conv_closure<float>(Executor&, const View& in, int H, int W, int C, const void* w,
                                                      float* scale, float* shift, int K, int R, int S, int sh,
                                                      int sw, int ph, int pw, int dh, int dw, int P, int Q, int relu,
                                                      const View& out, const std::vector<View>& out2, int& nk) {
  ConvSimtArgs a{};
  a.x = (const float*)in.p; a.H = H; a.W = W; a.C = C; a.ldx = in.ldc;
  a.w = (const float*)w; a.P = P; a.Q = Q; a.K = K; a.R = R; a.S = S; a.sh = sh; a.sw = sw; a.ph = ph;
  a.pw = pw; a.dh = dh; a.dw = dw; a.relu = relu; a.scale = scale; a.shift = shift;
  a.out = (float*)out.p; a.ldo = out.ldc;
  a.out2 = dst_of<float>(out2);
  nk += 1;
  return [a](cudaStream_t st) { launch_conv_simt(a, st); };
}

template <typename T>
static void build_op(Executor& ex, int v) {
  Graph& g = ex.g;
  const Op& o = g.ops[v];
  const int l = ex.s.gpu_of[v];
  OpExec& x = ex.ox[v];
  const int relu_v = (o.relu || ex.relu_out[v]) ? 1 : 0;  // the op's own ReLU, or its consumers' (hoisted)
  auto view_of = [&](int u, int on) { return View{ex.ptr(on, ex.loc[u][on].off), ex.loc[u][on].ldc}; };
  auto in_op = [&](int k) { return g.edges[o.in_edges[k]].src; };
  const View out = view_of(v, l);
  // fused remote destinations: every consumer GPU of a fusable op gets the
  // epilogue's stores directly (peer memory / aliased logical GPU)
  std::vector<View> out2;
  for (auto& r : x.remote)
    if (r.mode == DM_FUSED) out2.push_back(view_of(v, r.gpu));
  if (x.probe_out) out2.push_back(View{x.probe_out, x.probe_ldc});  // profiler: C15 edge probe
  std::vector<std::function<void(cudaStream_t)>> fns;
  int nk = 0;
  switch (o.kind) {
    case HIOS_OP_INPUT:
      break;  // staged before the graph (hios_run_device)
    case HIOS_OP_CONV: {
      const int u = in_op(0);
      const Op& xi = g.ops[u];
      // the conv's input: u's output, or (pre-ReLU conv) its ReLU'd copy --
      // made once after u on u's GPU (shared by every pre-ReLU consumer there)
      // or, for a remote / input producer, here into this op's scratch
      View cin = view_of(u, l);
      if (o.pre_relu && !ex.relu_out[u]) {
        auto it = ex.relu_loc.find((int64_t)u * ex.M + l);
        if (it != ex.relu_loc.end()) {
          cin = View{ex.ptr(l, it->second.off), it->second.ldc};
        } else {
          const View rv{ex.ptr(l, x.relubuf), x.relu_ldc};
          CopyArgs<T> c{(const T*)cin.p, cin.ldc, xi.H * xi.W, xi.C, (T*)rv.p, rv.ldc};
          fns.push_back([c](cudaStream_t st) { launch_relu_copy<T>(c, st); });
          ++nk;
          cin = rv;
        }
      }
      if (stem3_conv(o)) {
        View iv = cin;
        if (iv.ldc < (int)(16 / sizeof(T))) fail(HIOS_E_UNSUPPORTED, "stem input pixel pitch below 16 bytes");
        ConvStem3Args<T> c{};
        c.x = (const T*)iv.p; c.H = xi.H; c.W = xi.W; c.ldx = iv.ldc;
        c.P = o.H; c.Q = o.W; c.K = o.out_c; c.ph = o.ph; c.pw = o.pw; c.relu = relu_v;
        // whole 16-byte vectors (zeros into the pad channels) unless an output
        // is a concat slice, whose pad channels belong to the next producer
        bool own = true;
        for (int e : o.out_edges)
          if (ex.inplace[e]) own = false;
        c.kst = own ? rup(o.out_c, 8) : o.out_c;
        c.out = (T*)out.p; c.ldo = out.ldc;
        c.out2 = dst_of<T>(out2);
        auto wp = std::make_shared<Stem3W>();
        std::memset(wp.get(), 0, sizeof(Stem3W));
        for (int k = 0; k < o.out_c; ++k) {
          for (int cc = 0; cc < 3; ++cc)
            for (int r = 0; r < 3; ++r)
              for (int s2 = 0; s2 < 3; ++s2)
                wp->w[(r * 3 + s2) * 3 + cc][k] = o.weight[(((size_t)k * 3 + cc) * 3 + r) * 3 + s2];
          wp->scale[k] = o.scale[k];
          wp->shift[k] = o.shift[k];
        }
        fns.push_back([c, wp](cudaStream_t st) { launch_conv_stem3<T>(c, *wp, st); });
        ++nk;
        break;
      }
      if (x.s2dbuf >= 0) {
        View iv = cin;
        const int R2 = (o.kh + 1) / 2, S2 = (o.kw + 1) / 2;
        const int H2 = o.H + R2 - 1, W2 = o.W + S2 - 1;
        View sv{ex.ptr(l, x.s2dbuf), x.s2d_ldc};
        S2dArgs<T> d{(const T*)iv.p, xi.H, xi.W, xi.C, iv.ldc, o.ph, o.pw, (T*)sv.p, H2, W2, sv.ldc};
        fns.push_back([d](cudaStream_t st) { launch_s2d<T>(d, st); });
        ++nk;
        if (x.w_pack) {
          // packed taps: a virtual 64-channel input whose pixel j is the
          // 4-pixel window j..j+3 of the s2d tensor (pixel stride 32 B)
          View pv{sv.p, sv.ldc, W2};
          fns.push_back(conv_closure<T>(ex, pv, H2, o.W, 64, x.w_pack, x.scale[0], x.shift[0], o.out_c, R2, 1, 1, 1,
                                        0, 0, 1, 1, o.H, o.W, relu_v, out, out2, nk));
        } else {
          fns.push_back(conv_closure<T>(ex, sv, H2, W2, 4 * xi.C, x.w, x.scale[0], x.shift[0], o.out_c, R2, S2, 1, 1,
                                        0, 0, 1, 1, o.H, o.W, relu_v, out, out2, nk));
        }
        break;
      }
      if (small_c_conv(o)) {
        View iv = cin;
        ConvSmallArgs<T> c{};
        c.x = (const T*)iv.p; c.H = xi.H; c.W = xi.W; c.C = xi.C; c.ldx = iv.ldc;
        c.w = x.w_small; c.scale = x.scale[0]; c.shift = x.shift[0];
        c.P = o.H; c.Q = o.W; c.K = o.out_c; c.R = o.kh; c.S = o.kw; c.sh = o.sh; c.sw = o.sw;
        c.ph = o.ph; c.pw = o.pw; c.relu = relu_v;
        c.out = (T*)out.p; c.ldo = out.ldc;
        c.out2 = dst_of<T>(out2);
        fns.push_back([c](cudaStream_t st) { launch_conv_small_c<T>(c, st); });
        ++nk;
        break;
      }
      if (!g_conv_solo && ex.g.dtype == HIOS_BF16) {
        x.tc.clear();
        x.tc_smem = 0;
        g_tc_out = &x.tc;
        g_tc_smem = &x.tc_smem;
      }
      if (x.tap_r >= 0)  // single-tap conv: 1x1 on the tap-shifted input (same P x Q outputs)
        fns.push_back(conv_closure<T>(ex, cin, xi.H, xi.W, xi.C, x.w, x.scale[0], x.shift[0], o.out_c, 1, 1, o.sh,
                                      o.sw, o.ph - x.tap_r * o.dh, o.pw - x.tap_s * o.dw, 1, 1, o.H, o.W, relu_v, out,
                                      out2, nk));
      else
        fns.push_back(conv_closure<T>(ex, cin, xi.H, xi.W, xi.C, x.w, x.scale[0], x.shift[0], o.out_c, o.kh,
                                      o.kw, o.sh, o.sw, o.ph, o.pw, o.dh, o.dw, o.H, o.W, relu_v, out, out2, nk));
      g_tc_out = nullptr;
      g_tc_smem = nullptr;
      break;
    }
    case HIOS_OP_SEPCONV: {
      const Op& x0 = g.ops[in_op(0)];
      View dwv{ex.ptr(l, x.dwbuf), x.dw_ldc};
      View midv{x.midbuf >= 0 ? ex.ptr(l, x.midbuf) : nullptr, x.mid_ldc};
      for (int r = 0; r < o.reps; ++r) {
        DwArgs<T> d{};
        const int c = r == 0 ? o.in_c : o.out_c;
        const int Hi = r == 0 ? x0.H : o.H, Wi = r == 0 ? x0.W : o.W;
        if (r == 0) {
          const int nin = (int)o.in_edges.size();
          if (nin > HIOS_MAX_IN) fail(HIOS_E_UNSUPPORTED, "sepconv with more than 16 inputs");
          for (int k = 0; k < nin; ++k) {
            View iv = view_of(in_op(k), l);
            d.x[k] = (const T*)iv.p;
            d.ldx[k] = iv.ldc;
            d.agg[k] = o.agg.empty() ? 1.f : o.agg[k];
          }
          d.n_in = nin;
        } else {
          d.x[0] = (const T*)midv.p; d.ldx[0] = midv.ldc; d.agg[0] = 1.f; d.n_in = 1;
        }
        d.H = Hi; d.W = Wi; d.C = c; d.P = o.H; d.Q = o.W; d.R = o.kh; d.S = o.kw;
        d.sh = r == 0 ? o.sh : 1; d.sw = r == 0 ? o.sw : 1; d.ph = o.ph; d.pw = o.pw;
        d.pre_relu = o.pre_relu; d.w = x.dw[r]; d.out = (T*)dwv.p; d.ldo = dwv.ldc;
        fns.push_back([d](cudaStream_t st) { launch_dw<T>(d, st); });
        ++nk;
        const bool last = r == o.reps - 1;
        fns.push_back(conv_closure<T>(ex, dwv, o.H, o.W, c, x.pw[r], x.scale[r], x.shift[r], o.out_c, 1, 1, 1, 1, 0,
                                      0, 1, 1, o.H, o.W, last ? relu_v : 0, last ? out : midv,
                                      last ? out2 : std::vector<View>(), nk));
      }
      break;
    }
    case HIOS_OP_MAXPOOL:
    case HIOS_OP_AVGPOOL: {
      const int u = in_op(0);
      const Op& xi = g.ops[u];
      View iv = view_of(u, l);
      PoolArgs<T> p{};
      p.x = (const T*)iv.p; p.H = xi.H; p.W = xi.W; p.C = xi.C; p.ldx = iv.ldc;
      p.P = o.H; p.Q = o.W; p.kh = o.kh; p.kw = o.kw; p.sh = o.sh; p.sw = o.sw; p.ph = o.ph; p.pw = o.pw;
      p.is_max = o.kind == HIOS_OP_MAXPOOL; p.cip = o.cip;
      p.out = (T*)out.p; p.ldo = out.ldc;
      p.out2 = dst_of<T>(out2);
      fns.push_back([p](cudaStream_t st) { launch_pool<T>(p, st); });
      ++nk;
      break;
    }
    case HIOS_OP_GAP: {
      const int u = in_op(0);
      const Op& xi = g.ops[u];
      View iv = view_of(u, l);
      const T* xp = (const T*)iv.p;
      const int HW = xi.H * xi.W, C = xi.C, ldx = iv.ldc;
      T* op = (T*)out.p;
      fns.push_back([=](cudaStream_t st) { launch_gap<T>(xp, HW, C, ldx, op, st); });
      ++nk;
      break;
    }
    case HIOS_OP_LINEAR: {
      View iv = view_of(in_op(0), l);
      const T* xp = (const T*)iv.p;
      const T* w = (const T*)x.w;
      const int Cin = o.in_c, K = o.out_c, ldw = x.ldw;
      const float* b = x.bias;
      T* op = (T*)out.p;
      fns.push_back([=](cudaStream_t st) { launch_linear<T>(xp, Cin, w, ldw, b, K, op, st); });
      ++nk;
      break;
    }
    case HIOS_OP_CONCAT: {
      int c_off = 0;
      for (int e : o.in_edges) {
        const int u = g.edges[e].src;
        const Op& xu = g.ops[u];
        if (!ex.inplace[e]) {
          View iv = view_of(u, l);
          CopyArgs<T> c{(const T*)iv.p, iv.ldc, o.H * o.W, xu.C, (T*)(out.p + (size_t)c_off * ex.esz), out.ldc};
          // a ReLU'd concat (relu_out) whose input keeps its raw output: ReLU'd slice copy
          if (ex.relu_out[v] && !ex.relu_out[u]) fns.push_back([c](cudaStream_t st) { launch_relu_copy<T>(c, st); });
          else fns.push_back([c](cudaStream_t st) { launch_copy<T>(c, st); });
          ++nk;
        }
        c_off += xu.C;
      }
      break;
    }
    case HIOS_OP_ADD: {
      const int nin = (int)o.in_edges.size();
      if (nin > HIOS_MAX_IN) fail(HIOS_E_UNSUPPORTED, "add with more than 16 inputs");
      AddArgs<T> a{};
      for (int k = 0; k < nin; ++k) {
        View iv = view_of(in_op(k), l);
        a.x[k] = (const T*)iv.p; a.ldx[k] = iv.ldc; a.agg[k] = o.agg[k];
      }
      a.n_in = nin; a.HW = o.H * o.W; a.C = o.C; a.relu = relu_v;
      a.out = (T*)out.p; a.ldo = out.ldc;
      a.out2 = dst_of<T>(out2);
      fns.push_back([a](cudaStream_t st) { launch_add<T>(a, st); });
      ++nk;
      break;
    }
    case HIOS_OP_IDENTITY: {
      View iv = view_of(in_op(0), l);
      CopyArgs<T> c{(const T*)iv.p, iv.ldc, o.H * o.W, o.C, (T*)out.p, out.ldc};
      if (relu_v) fns.push_back([c](cudaStream_t st) { launch_relu_copy<T>(c, st); });
      else fns.push_back([c](cudaStream_t st) { launch_copy<T>(c, st); });
      ++nk;
      break;
    }
  }
  {  // ReLU'd copy of this op's output for the pre-ReLU convs that read it here
    auto it = ex.relu_loc.find((int64_t)v * ex.M + l);
    if (it != ex.relu_loc.end()) {
      CopyArgs<T> c{(const T*)out.p, out.ldc, o.H * o.W, o.C, (T*)ex.ptr(l, it->second.off), it->second.ldc};
      fns.push_back([c](cudaStream_t st) { launch_relu_copy<T>(c, st); });
      ++nk;
    }
  }
  x.run = [fns](cudaStream_t st) {
    for (auto& f : fns) f(st);
  };
  x.n_kernels = nk;
}

void Executor::build_op_closures(int v) {
  const int l = s.gpu_of[v];
  ck(cudaSetDevice(lg[l].dev), "cudaSetDevice");
  cur_lgpu = l;
  g_num_sms = lg[l].num_sms;
  OpExec& x = ox[v];
  g_plan_out = x.plan;
  if (g.dtype == HIOS_BF16) build_op<bf16>(*this, v);
  else build_op<float>(*this, v);
  g_plan_out = nullptr;
  const int k = g.ops[v].kind;
  if (g.dtype == HIOS_BF16 && (k == HIOS_OP_CONV || k == HIOS_OP_SEPCONV)) {
    auto run = x.run;
    const int nk = x.n_kernels;
    auto tc = x.tc;
    const size_t tcs = x.tc_smem;
    g_conv_solo = true;
    g_plan_out = x.plan_solo;
    build_op<bf16>(*this, v);
    g_plan_out = nullptr;
    g_conv_solo = false;
    x.run_solo = x.run;
    x.n_kernels_solo = x.n_kernels;
    x.run = run;
    x.n_kernels = nk;
    x.tc = tc;
    x.tc_smem = tcs;
  }
}

void Executor::build_closures() {
  for (int v = 0; v < g.n; ++v)
    if (lg[s.gpu_of[v]].local) build_op_closures(v);
}

// deliveries of op u's output to other logical GPUs: push (unless fused) + flag release
static int enqueue_deliver(Executor& ex, int u, cudaStream_t st) {
  const int l = ex.s.gpu_of[u];
  const Op& o = ex.g.ops[u];
  int nk = 0;
  for (auto& r : ex.ox[u].remote) {
    const int d = r.gpu;
    if (r.mode == DM_NCCL) {
      // pack into the send staging buffer if needed; the send itself is
      // posted on the communication stream in the global order
      for (auto& x : ex.xfers) {
        if (x.u != u || x.dst != d) continue;
        if (x.send_off >= 0) {
          const Loc& src = ex.loc[u][l];
          if (ex.g.dtype == HIOS_BF16) {
            CopyArgs<bf16> c{(const bf16*)ex.ptr(l, src.off), src.ldc, o.H * o.W, o.C, (bf16*)ex.ptr(l, x.send_off), o.C};
            launch_copy<bf16>(c, st);
          } else {
            CopyArgs<float> c{(const float*)ex.ptr(l, src.off), src.ldc, o.H * o.W, o.C, (float*)ex.ptr(l, x.send_off),
                              o.C};
            launch_copy<float>(c, st);
          }
          ++nk;
        }
        ck(cudaEventRecord(x.ev_ready, st), "record send-ready");
      }
      continue;
    }
    if (r.mode == DM_COPY) {
      // copy-engine transfer after the producer finished (the paper's
      // "launch after the transfer completes" design): a strided
      // 2-D copy (C channels per pixel, pixel pitches of both buffers)
      const Loc& src = ex.loc[u][l];
      const Loc& dst = ex.loc[u][d];
      ck(cudaMemcpy2DAsync(ex.ptr(d, dst.off), (size_t)dst.ldc * ex.esz, ex.ptr(l, src.off), (size_t)src.ldc * ex.esz,
                           (size_t)o.C * ex.esz, (size_t)o.H * o.W, cudaMemcpyDefault, st),
         "cudaMemcpy2DAsync (copy transport)");
    } else if (r.mode == DM_PUSH) {
      const Loc& src = ex.loc[u][l];
      const Loc& dst = ex.loc[u][d];
      if (ex.g.dtype == HIOS_BF16) {
        CopyArgs<bf16> c{(const bf16*)ex.ptr(l, src.off), src.ldc, o.H * o.W, o.C, (bf16*)ex.ptr(d, dst.off), dst.ldc};
        launch_copy<bf16>(c, st);
      } else {
        CopyArgs<float> c{(const float*)ex.ptr(l, src.off), src.ldc, o.H * o.W, o.C, (float*)ex.ptr(d, dst.off),
                          dst.ldc};
        launch_copy<float>(c, st);
      }
      ++nk;
    }
    if (ex.same_graph(l, d)) {
      // consumer in the same CUDA graph (a logical GPU aliased on this
      // device): a graph dependency, no device-side flag
      ck(cudaEventRecord(ex.edge_event(u, d), st), "record edge");
    } else {
      launch_signal(ex.lg[l].sync, ex.lg[d].sync + 1 + ex.M + ex.flag_index[u][d], st);
      ++nk;
    }
  }
  return nk;
}

// SM partition of a stage's grouped convs: op i gets n_i persistent CTAs (one
// per SM) and runs ceil(T_i / n_i) rounds of tiles, each ~tau_i (its measured
// solo time per round of tiles).  Greedy makespan minimisation: start at one
// CTA each, repeatedly give the op with the latest finish the smallest number
// of extra CTAs that removes one of its rounds, while the budget lasts.  SMs
// the convs cannot use stay free for the stage's other ops.
static std::vector<int> partition_ctas(const std::vector<int>& tiles, const std::vector<double>& tau, int budget) {
  const int n = (int)tiles.size();
  std::vector<int> c(n, 1);
  int used = n;
  auto rounds = [&](int i, int k) { return (tiles[i] + k - 1) / k; };
  while (true) {
    int j = -1;
    double worst = -1;
    for (int i = 0; i < n; ++i) {
      const double f = rounds(i, c[i]) * tau[i];
      if (f > worst) { worst = f; j = i; }
    }
    const int r = rounds(j, c[j]);
    if (r <= 1) break;  // the latest op already runs in one round
    const int need = (tiles[j] + r - 2) / (r - 1);  // fewest CTAs giving r - 1 rounds
    if (used + need - c[j] > budget) break;
    used += need - c[j];
    c[j] = need;
  }
  return c;
}

void Executor::enqueue_stage(int l, const std::vector<int>& S, bool timed, int64_t& nk,
                             const std::function<void(int, cudaStream_t)>& post, cudaStream_t lane,
                             bool singleton) {
  LGpu& L = lg[l];
  cudaStream_t s0 = lane ? lane : L.streams[0];
  auto run_one = [&](int v, cudaStream_t st) {
    if (timed) ck(cudaEventRecordWithFlags(op_ev0[v], st, cudaEventRecordExternal), "event record");
    const bool solo = singleton && S.size() == 1 && ox[v].run_solo;
    (solo ? ox[v].run_solo : ox[v].run)(st);
    if (timed) ck(cudaEventRecordWithFlags(op_ev1[v], st, cudaEventRecordExternal), "event record");
    nk += solo ? ox[v].n_kernels_solo : ox[v].n_kernels;
    post(v, st);
  };
  if (S.size() == 1) {
    run_one(S[0], s0);
    return;
  }
  std::vector<int> grp, rest;
  for (int v : S) (group_convs && ox[v].tc.size() == 1 ? grp : rest).push_back(v);
  if (grp.size() < 2 || (int)grp.size() > kMaxGroup) {
    grp.clear();
    rest = S;
  }
  const int n_streams_used = (int)rest.size() + (grp.empty() ? 0 : 1);
  if (n_streams_used > 1) {
    ck(cudaEventRecord(L.ev_fork, s0), "fork");
    for (int k = 1; k < n_streams_used; ++k) ck(cudaStreamWaitEvent(L.streams[k], L.ev_fork, 0), "fork wait");
  }
  int k0 = 0;
  if (!grp.empty()) {
    // one launch for the stage's convs; the non-conv ops of the stage keep
    // a share of the SMs proportional to their measured time
    double wc = 0, wr = 0;
    std::vector<int> tiles;
    std::vector<double> tau;
    for (int v : grp) {
      const ConvTcArgs& a = ox[v].tc[0].a;
      const int T = a.tiles_m * a.tiles_n;
      tiles.push_back(T);
      const double w = g.ops[v].cost > 0 ? (double)g.ops[v].cost : 1.0;
      tau.push_back(w / ((T + L.num_sms - 1) / L.num_sms));  // per round of tiles
      wc += w;
    }
    for (int v : rest) wr += g.ops[v].cost > 0 ? (double)g.ops[v].cost : 1.0;
    int budget = L.num_sms;
    if (!rest.empty())
      budget = std::max((int)grp.size(), std::min(L.num_sms - 16, (int)std::lround(L.num_sms * wc / (wc + wr))));
    const std::vector<int> c = partition_ctas(tiles, tau, budget);
    ConvTcGroup G;
    std::memset(&G, 0, sizeof(G));
    G.n = (int)grp.size();
    size_t smem = 0;
    for (int i = 0; i < G.n; ++i) {
      G.op[i] = ox[grp[i]].tc[0];
      G.cta0[i + 1] = G.cta0[i] + c[i];
      smem = std::max(smem, ox[grp[i]].tc_smem);
    }
    if (timed)
      for (int v : grp) ck(cudaEventRecordWithFlags(op_ev0[v], s0, cudaEventRecordExternal), "event record");
    launch_conv_tc_group(G, smem, s0);
    ++nk;
    if (timed)
      for (int v : grp) ck(cudaEventRecordWithFlags(op_ev1[v], s0, cudaEventRecordExternal), "event record");
    for (int v : grp) post(v, s0);
    k0 = 1;
  }
  for (size_t i = 0; i < rest.size(); ++i) run_one(rest[i], L.streams[k0 + i]);
  for (int k = 1; k < n_streams_used; ++k) {
    ck(cudaEventRecord(L.ev_join[k], L.streams[k]), "join");
    ck(cudaStreamWaitEvent(s0, L.ev_join[k], 0), "join wait");
  }
}

// The stage programs of the local logical GPUs that share one device, captured
// into ONE CUDA graph.  Several logical GPUs alias one device when a schedule
// has more GPUs than the box; edges between them become graph dependencies
// (event record -> stream wait inside the capture), not device-side flag
// spins (a spinning wait kernel could block the hardware queue its signaller
// sits behind).  Edges to other devices / processes keep the epoch flags
// (peer / copy transports) or the NCCL send / receive pairs.  The stages of
// all logical GPUs of the graph are captured in one topological order of the
// stage DAG (the same order the NCCL transport posts its transfers in).
void Executor::capture_device(const std::vector<int>& ls, bool timed) {
  const std::set<int> lset(ls.begin(), ls.end());
  const int l0 = ls[0];
  LGpu& L0 = lg[l0];
  cudaStream_t origin = L0.streams[0];
  int64_t nk = 0;
  ck(cudaStreamBeginCapture(origin, cudaStreamCaptureModeRelaxed), "begin capture");
  if (ls.size() > 1) {
    ck(cudaEventRecord(L0.ev_fork, origin), "fork lgpus");
    for (size_t i = 1; i < ls.size(); ++i) ck(cudaStreamWaitEvent(lg[ls[i]].streams[0], L0.ev_fork, 0), "fork");
  }
  std::set<std::pair<int, int>> acks_out;  // (this lgpu, producer lgpu in another graph)
  for (int l : ls) {
    LGpu& L = lg[l];
    cudaStream_t s0 = L.streams[0];
    launch_epoch(L.sync, s0);
    ++nk;
    // back-pressure: do not overwrite a consumer GPU's buffers (in another
    // graph) before it finished the previous run
    std::set<int> consumers;
    for (int v = 0; v < g.n; ++v) {
      if (s.gpu_of[v] == l) {
        for (auto& r : ox[v].remote)
          if (r.mode != DM_NCCL && !lset.count(r.gpu)) consumers.insert(r.gpu);
      } else if (flag_index[v][l] >= 0 && !lset.count(s.gpu_of[v])) {
        acks_out.insert({l, s.gpu_of[v]});
      }
    }
    for (int c : consumers) {
      launch_wait(L.sync, L.sync + 1 + c, 1, s0);
      ++nk;
    }
  }
  // NCCL: this device's sends / receives in the global transfer order on one
  // communication stream (forked from and joined back into the origin)
  std::vector<int> acts;
  for (int k = 0; k < (int)xfers.size(); ++k)
    if (lset.count(xfers[k].src) || lset.count(xfers[k].dst)) acts.push_back(k);
  size_t next = 0;
  std::vector<char> ready(xfers.size(), 0);
  cudaStream_t cs = L0.comm;
  if (!acts.empty()) {
    ck(cudaEventRecord(L0.ev_fork, origin), "fork comm");
    ck(cudaStreamWaitEvent(cs, L0.ev_fork, 0), "fork comm wait");
  }
  auto post = [&](size_t upto) {
    for (; next < upto; ++next) {
      NcclXfer& x = xfers[acts[next]];
      const Op& o = g.ops[x.u];
      if (lset.count(x.src)) {
        if (!ready[acts[next]])
          fail(HIOS_E_STATE, "NCCL transfer order inconsistent with the stage order (op " + std::to_string(x.u) + ")");
        ck(cudaStreamWaitEvent(cs, x.ev_ready, 0), "wait send-ready");
        const void* p = x.send_off >= 0 ? ptr(x.src, x.send_off) : ptr(x.src, loc[x.u][x.src].off);
        nccl_send(p, x.bytes, s.owner[x.dst], comm, cs);
      } else {
        const int l = x.dst;
        void* p = x.recv_off >= 0 ? ptr(l, x.recv_off) : ptr(l, loc[x.u][l].off);
        nccl_recv(p, x.bytes, s.owner[x.src], comm, cs);
        if (x.recv_off >= 0) {  // unpack into the consumer's location (slice / pitch)
          const Loc& dl = loc[x.u][l];
          if (g.dtype == HIOS_BF16) {
            CopyArgs<bf16> c{(const bf16*)p, o.C, o.H * o.W, o.C, (bf16*)ptr(l, dl.off), dl.ldc};
            launch_copy<bf16>(c, cs);
          } else {
            CopyArgs<float> c{(const float*)p, o.C, o.H * o.W, o.C, (float*)ptr(l, dl.off), dl.ldc};
            launch_copy<float>(c, cs);
          }
          ++nk;
        }
        ck(cudaEventRecord(x.ev_recv, cs), "record recv");
      }
    }
  };
  // every stage of the graph's logical GPUs in one topological order
  const std::vector<std::vector<int>> rank = stage_ranks(s);
  std::vector<std::tuple<int, int, int>> order;
  for (int l : ls)
    for (int j = 0; j < (int)s.Q[l].size(); ++j) order.emplace_back(rank[l][j], l, j);
  std::sort(order.begin(), order.end());
  cur_graph = lset;
  // a cross-GPU input u of an op on logical GPU l, waited for on stream st
  auto wait_remote = [&](int u, int l, cudaStream_t st) {
    const int p = s.gpu_of[u];
    if (lset.count(p)) {
      ck(cudaStreamWaitEvent(st, edge_event(u, l), 0), "wait edge");
    } else if (flag_index[u][l] < 0) {  // NCCL: post up to this receive, then wait for it
      for (size_t i = 0; i < acts.size(); ++i) {
        const NcclXfer& x = xfers[acts[i]];
        if (x.u == u && x.dst == l) {
          post(std::max(next, i + 1));
          ck(cudaStreamWaitEvent(st, x.ev_recv, 0), "wait recv");
        }
      }
    } else {
      launch_wait(lg[l].sync, lg[l].sync + 1 + M + flag_index[u][l], 0, st);
      ++nk;
    }
  };
  auto deliver = [&](int v, cudaStream_t st) {
    nk += enqueue_deliver(*this, v, st);
    for (int k : acts)
      if (xfers[k].u == v && lset.count(xfers[k].src)) ready[k] = 1;
  };
  // dataflow stage mode: op i of a stage runs on lane (stream) i and waits only
  // for its own inputs (done events of same-GPU producers on other lanes) and
  // the previous op of its lane -- no join at the stage boundary
  std::vector<char> lanes_forked(M, 0);
  std::vector<std::vector<double>> lane_free(M);  // dataflow: predicted time each lane is free
  std::vector<std::vector<int>> lane_last(M);     // dataflow: last op on each lane
  std::vector<double> pred_fin(g.n, 0.0);         // dataflow: predicted finish of op v
  for (int l : ls) {
    lane_free[l].assign(lg[l].streams.size(), 0.0);
    lane_last[l].assign(lg[l].streams.size(), -1);
  }
  std::fill(lane_of.begin(), lane_of.end(), -1);
  for (auto& it : order) {
    const int l = std::get<1>(it), j = std::get<2>(it);
    LGpu& L = lg[l];
    cudaStream_t s0 = L.streams[0];
    const auto& S = s.Q[l][j];
    if (dataflow) {
      if (!lanes_forked[l]) {
        lanes_forked[l] = 1;
        ck(cudaEventRecord(L.ev_fork, s0), "fork lanes");
        for (size_t k = 1; k < L.streams.size(); ++k) ck(cudaStreamWaitEvent(L.streams[k], L.ev_fork, 0), "fork");
      }
      // lane choice (list scheduling on the measured t(v)): the lane whose
      // last op is v's latest-finishing same-GPU producer (the stream order is
      // then a real dependency), else the lane free earliest; one lane per op
      // of the stage
      std::vector<char> taken(L.streams.size(), 0);
      for (size_t i = 0; i < S.size(); ++i) {
        const int v = S[i];
        std::set<int> ins;
        for (int e : g.ops[v].in_edges) ins.insert(g.edges[e].src);
        double ready = 0;
        int prod_lane = -1;
        double prod_fin = -1;
        for (int u : ins)
          if (s.gpu_of[u] == l && lane_of[u] >= 0) {
            ready = std::max(ready, pred_fin[u]);
            if (pred_fin[u] > prod_fin && lane_last[l][lane_of[u]] == u && !taken[lane_of[u]]) {
              prod_fin = pred_fin[u];
              prod_lane = lane_of[u];
            }
          }
        int k = prod_lane;
        if (k < 0) {
          for (size_t c = 0; c < L.streams.size(); ++c)
            if (!taken[c] && (k < 0 || lane_free[l][c] < lane_free[l][k])) k = (int)c;
        }
        taken[k] = 1;
        cudaStream_t st = L.streams[k];
        for (int u : ins) {
          if (s.gpu_of[u] != l) wait_remote(u, l, st);
          else if (g.ops[u].kind != HIOS_OP_INPUT && !(lane_of[u] == k && lane_last[l][k] == u))
            ck(cudaStreamWaitEvent(st, done_ev[u], 0), "wait input");
        }
        enqueue_stage(l, std::vector<int>{v}, timed, nk, deliver, st, S.size() == 1);
        ck(cudaEventRecord(done_ev[v], st), "done");
        lane_of[v] = k;
        lane_last[l][k] = v;
        const double t = std::max<double>(1.0, (double)g.ops[v].cost);
        pred_fin[v] = std::max(ready, lane_free[l][k]) + t;
        lane_free[l][k] = pred_fin[v];
      }
      continue;
    }
    std::set<int> waits;
    for (int v : S)
      for (int e : g.ops[v].in_edges) {
        const int u = g.edges[e].src;
        if (s.gpu_of[u] != l) waits.insert(u);
      }
    for (int u : waits) wait_remote(u, l, s0);
    enqueue_stage(l, S, timed, nk, deliver);
  }
  if (dataflow)
    for (int l : ls) {
      LGpu& L = lg[l];
      if (!lanes_forked[l]) continue;
      for (size_t k = 1; k < L.streams.size(); ++k) {
        ck(cudaEventRecord(L.ev_join[k], L.streams[k]), "join lane");
        ck(cudaStreamWaitEvent(L.streams[0], L.ev_join[k], 0), "join lane wait");
      }
    }
  cur_graph.clear();
  if (!acts.empty()) {
    post(acts.size());
    ck(cudaEventRecord(L0.ev_join[0], cs), "join comm");
    ck(cudaStreamWaitEvent(origin, L0.ev_join[0], 0), "join comm wait");
  }
  for (auto& pr : acks_out) {
    launch_signal(lg[pr.first].sync, lg[pr.second].sync + 1 + pr.first, lg[pr.first].streams[0]);
    ++nk;
  }
  for (size_t i = 1; i < ls.size(); ++i) {
    LGpu& L = lg[ls[i]];
    ck(cudaEventRecord(L.ev_join[0], L.streams[0]), "join lgpu");
    ck(cudaStreamWaitEvent(origin, L.ev_join[0], 0), "join lgpu wait");
  }
  cudaGraph_t graph;
  ck(cudaStreamEndCapture(origin, &graph), "end capture");
  cudaGraphExec_t ge;
  ck(cudaGraphInstantiate(&ge, graph, 0), "graph instantiate");
  cudaGraphDestroy(graph);
  (timed ? L0.gexec_timed : L0.gexec) = ge;
  if (!timed) kernels_per_run += nk;
}

cudaEvent_t Executor::edge_event(int u, int d) {
  auto it = edge_ev.find((int64_t)u * M + d);
  if (it == edge_ev.end()) fail(HIOS_E_STATE, "no edge event");
  return it->second;
}

void Executor::capture() {
  if (op_ev0.empty()) {
    op_ev0.assign(g.n, nullptr);
    op_ev1.assign(g.n, nullptr);
    done_ev.assign(g.n, nullptr);
    lane_of.assign(g.n, -1);
  }
  kernels_per_run = 0;
  for (int l = 0; l < M; ++l) {
    LGpu& L = lg[l];
    if (!L.local) continue;
    ck(cudaSetDevice(L.dev), "cudaSetDevice");
    for (int v = 0; v < g.n; ++v)
      if (s.gpu_of[v] == l && !op_ev0[v]) {
        ck(cudaEventCreate(&op_ev0[v]), "event");
        ck(cudaEventCreate(&op_ev1[v]), "event");
        ck(cudaEventCreateWithFlags(&done_ev[v], cudaEventDisableTiming), "event");
      }
  }
  // HIOS_STAGE_AUTO (one process driving all its GPUs): the dataflow variant
  // is captured first and parked in gexec*_alt, then the streams variant
  const bool both = auto_pending && std::all_of(lg.begin(), lg.end(), [](const LGpu& L) { return L.local; });
  if (!both) auto_pending = false;
  for (int pass = both ? 0 : 1; pass < 2; ++pass) {
    dataflow = pass == 0 ? true : (both ? false : dataflow);
    const int64_t kpr = kernels_per_run;
    for (auto& kv : graphs_by_dev) {
      ck(cudaSetDevice(kv.first), "cudaSetDevice");
      for (int timed = 0; timed < 2; ++timed) capture_device(kv.second, timed != 0);
      if (pass == 0) {
        LGpu& L0 = lg[kv.second[0]];
        std::swap(L0.gexec, L0.gexec_alt);
        std::swap(L0.gexec_timed, L0.gexec_timed_alt);
      }
    }
    if (pass == 0) kernels_per_run = kpr;  // counted once (the variants launch the same kernels)
  }
  captured = true;
}

// HIOS_STAGE_AUTO: replay both captured variants (graphs only, on the arena's
// current contents) and keep the faster; wall time of launch-all + sync-all,
// median of 7 after 2 warm-ups each.
void Executor::choose_variant() {
  auto run_all = [&](bool alt) {
    const auto t0 = std::chrono::steady_clock::now();
    for (auto& kv : graphs_by_dev) {
      LGpu& L = lg[kv.second[0]];
      ck(cudaSetDevice(L.dev), "cudaSetDevice");
      ck(cudaGraphLaunch(alt ? L.gexec_alt : L.gexec, L.streams[0]), "graph launch");
    }
    for (auto& kv : graphs_by_dev) {
      LGpu& L = lg[kv.second[0]];
      ck(cudaSetDevice(L.dev), "cudaSetDevice");
      ck(cudaStreamSynchronize(L.streams[0]), "synchronize");
    }
    return std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  };
  double med[2];
  for (int alt = 0; alt < 2; ++alt) {
    std::vector<double> t;
    for (int i = 0; i < 9; ++i) {
      const double x = run_all(alt != 0);
      if (i >= 2) t.push_back(x);
    }
    std::sort(t.begin(), t.end());
    med[alt] = t[t.size() / 2];
  }
  if (med[1] < med[0]) {
    for (auto& kv : graphs_by_dev) {
      LGpu& L = lg[kv.second[0]];
      std::swap(L.gexec, L.gexec_alt);
      std::swap(L.gexec_timed, L.gexec_timed_alt);
    }
    mode_used = HIOS_STAGE_DATAFLOW;
  } else {
    mode_used = HIOS_STAGE_STREAMS;
  }
  auto_pending = false;
}

void Executor::run_device(const void* d_in, void* d_out, cudaStream_t user, bool timed) {
  if (!lowered) {
    plan();
    allocate();
  }
  if (!captured) {
    build_closures();
    capture();
  }
  int cur = 0;
  ck(cudaGetDevice(&cur), "cudaGetDevice");
  cudaEvent_t ev_user = nullptr;
  if (user) {
    ck(cudaEventCreateWithFlags(&ev_user, cudaEventDisableTiming), "event");
    ck(cudaEventRecord(ev_user, user), "record user");
  }
  const int li = s.gpu_of[g.input_op], lsk = s.gpu_of[g.sink_op];
  for (auto& kv : graphs_by_dev) {
    const int o = kv.second[0];
    LGpu& L = lg[o];
    ck(cudaSetDevice(L.dev), "cudaSetDevice");
    if (ev_user) ck(cudaStreamWaitEvent(L.streams[0], ev_user, 0), "wait user");
    ck(cudaEventRecord(L.ev_start, L.streams[0]), "record start");
    if (graph_of[li] == o && d_in) {
      const Loc& lc = loc[g.input_op][li];
      if (g.dtype == HIOS_BF16)
        launch_input<bf16>((const float*)d_in, g.in_c, g.in_h, g.in_w, (bf16*)ptr(li, lc.off), lc.ldc, L.streams[0]);
      else
        launch_input<float>((const float*)d_in, g.in_c, g.in_h, g.in_w, (float*)ptr(li, lc.off), lc.ldc,
                            L.streams[0]);
    }
  }
  for (auto& kv : graphs_by_dev) {
    LGpu& L = lg[kv.second[0]];
    ck(cudaSetDevice(L.dev), "cudaSetDevice");
    ck(cudaGraphLaunch(timed ? L.gexec_timed : L.gexec, L.streams[0]), "graph launch");
  }
  for (auto& kv : graphs_by_dev) {
    const int o = kv.second[0];
    LGpu& L = lg[o];
    ck(cudaSetDevice(L.dev), "cudaSetDevice");
    if (graph_of[lsk] == o && d_out) {
      const Op& op = g.ops[g.sink_op];
      const Loc& lc = loc[g.sink_op][lsk];
      if (g.dtype == HIOS_BF16)
        launch_output<bf16>((const bf16*)ptr(lsk, lc.off), op.C, op.H, op.W, lc.ldc, (float*)d_out, L.streams[0]);
      else
        launch_output<float>((const float*)ptr(lsk, lc.off), op.C, op.H, op.W, lc.ldc, (float*)d_out, L.streams[0]);
    }
    ck(cudaEventRecord(L.ev_done, L.streams[0]), "record done");
  }
  ck(cudaSetDevice(cur), "cudaSetDevice");
  for (auto& kv : graphs_by_dev) {
    LGpu& L = lg[kv.second[0]];
    if (user) ck(cudaStreamWaitEvent(user, L.ev_done, 0), "user wait");
    else ck(cudaEventSynchronize(L.ev_done), "synchronize");
  }
  if (ev_user) cudaEventDestroy(ev_user);
  ck(cudaGetLastError(), "run");
  if (auto_pending) {
    // the first run's results stand; the variants are then timed on its data
    for (auto& kv : graphs_by_dev) {
      ck(cudaSetDevice(lg[kv.second[0]].dev), "cudaSetDevice");
      ck(cudaStreamSynchronize(lg[kv.second[0]].streams[0]), "synchronize");
    }
    choose_variant();
    ck(cudaSetDevice(cur), "cudaSetDevice");
  }
}

// Uninstrumented per-op device time of the schedule's own kernels (bench.py's
// roofline): for op v, one CUDA graph = [L2 flush (a write of flush_bytes) ->
// event -> v's kernels as configured in Q (its stage context) -> event],
// replayed reps + 1 times (the first is a warm-up); median of the event
// intervals.  Cold L2 per op, like ncu's default --cache-control all.
void Executor::time_ops(int reps, int64_t flush_bytes, int64_t* op_ns) {
  if (!lowered) {
    plan();
    allocate();
  }
  if (!captured) {
    build_closures();
    capture();
  }
  for (int v = 0; v < g.n; ++v) op_ns[v] = -1;
  for (int l = 0; l < M; ++l) {
    LGpu& L = lg[l];
    if (!L.local) continue;
    ck(cudaSetDevice(L.dev), "cudaSetDevice");
    void* fl = nullptr;
    if (flush_bytes > 0) ck(cudaMalloc(&fl, (size_t)flush_bytes), "cudaMalloc flush");
    cudaEvent_t a, b;
    ck(cudaEventCreate(&a), "event");
    ck(cudaEventCreate(&b), "event");
    cudaStream_t st = L.streams[0];
    for (int j = 0; j < (int)s.Q[l].size(); ++j) {
      const auto& S = s.Q[l][j];
      for (int v : S) {
        if (g.ops[v].kind == HIOS_OP_INPUT || g.ops[v].kind == HIOS_OP_CONCAT) continue;
        const bool solo = S.size() == 1 && ox[v].run_solo;
        cudaGraph_t graph;
        ck(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed), "time_ops capture");
        if (fl) launch_fill(fl, (size_t)flush_bytes, st);
        ck(cudaEventRecordWithFlags(a, st, cudaEventRecordExternal), "record");
        (solo ? ox[v].run_solo : ox[v].run)(st);
        ck(cudaEventRecordWithFlags(b, st, cudaEventRecordExternal), "record");
        ck(cudaStreamEndCapture(st, &graph), "time_ops capture end");
        cudaGraphExec_t ge;
        ck(cudaGraphInstantiate(&ge, graph, 0), "time_ops instantiate");
        cudaGraphDestroy(graph);
        std::vector<float> ms;
        for (int i = 0; i <= std::max(1, reps); ++i) {
          ck(cudaGraphLaunch(ge, st), "time_ops launch");
          ck(cudaStreamSynchronize(st), "time_ops sync");
          float t = 0;
          ck(cudaEventElapsedTime(&t, a, b), "elapsed");
          if (i > 0) ms.push_back(t);
        }
        cudaGraphExecDestroy(ge);
        std::sort(ms.begin(), ms.end());
        op_ns[v] = (int64_t)(ms[ms.size() / 2] * 1e6);
      }
    }
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    if (fl) cudaFree(fl);
  }
}

void Executor::read_output(int op, float* host, int64_t n) {
  const int l = s.gpu_of[op];
  if (!lg[l].local) fail(HIOS_E_INVALID, "op not executed by this process");
  const Op& o = g.ops[op];
  if (n < (int64_t)o.C * o.H * o.W) fail(HIOS_E_INVALID, "output buffer too small");
  ck(cudaSetDevice(lg[l].dev), "cudaSetDevice");
  float* tmp = nullptr;
  const size_t bytes = (size_t)o.C * o.H * o.W * sizeof(float);
  ck(cudaMalloc(&tmp, bytes), "cudaMalloc");
  const Loc& lc = loc[op][l];
  cudaStream_t st = lg[l].streams[0];
  if (g.dtype == HIOS_BF16)
    launch_output<bf16>((const bf16*)ptr(l, lc.off), o.C, o.H, o.W, lc.ldc, tmp, st);
  else
    launch_output<float>((const float*)ptr(l, lc.off), o.C, o.H, o.W, lc.ldc, tmp, st);
  ck(cudaStreamSynchronize(st), "sync");
  ck(cudaMemcpy(host, tmp, bytes, cudaMemcpyDeviceToHost), "D2H");
  cudaFree(tmp);
}

}  // namespace hios
