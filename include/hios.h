/*
 * hios.h -- C-ABI of the B200-native HIOS executor.
 *
 * The calls follow the problem statement of Kundu & Shu, "HIOS: Hierarchical
 * Inter-Operator Scheduler ..." (IEEE CLUSTER 2023); P:<line> cites
 * /root/reference/PAPER.md.
 *
 *   Given  the computation graph G = (V, E), M homogeneous GPUs, the execution
 *          time t(S) of each set S of <= K independent operators on one GPU and
 *          the communication time t(u, v) ...
 *   Find   a feasible schedule Q minimizing the inference latency
 *          subject to t^S(S_{i',j'}) - t^F(S_{i,j}) >= t(u,v) if i != i'
 *          (>= 0 on one GPU), for all (u, v) in E
 *
 *   hios_graph_create  -- G: ops = vertices, edges = tensors u -> v
 *   hios_profile       -- t(v), t(u, v) measured on device; t(S) measured
 *                         lazily (memoised) when the scheduler asks
 *   hios_schedule_lp   -- HIOS-LP: Alg. 1 (iterative longest-path mapping,
 *                         P:124-140) + Alg. 2 (sliding window)
 *   hios_run           -- batch-1 inference under Q on the GPUs
 *
 * Conventions (all calls):
 *   - Every call returns a hios_status; HIOS_OK = 0.  On failure nothing the
 *     caller owns is modified, *out handles are set to NULL, and
 *     hios_last_error() returns a thread-local message valid until the next
 *     call on that thread.  No exception or abort crosses the ABI.
 *   - All caller arrays are copied; the caller may free them after the call.
 *   - Handles are not thread-safe; one thread at a time per handle.
 *   - Costs are int64 nanoseconds.  A negative cost means "unknown".
 *   - Tensors at the ABI are fp32, NCHW, batch 1.  On device the executor
 *     stores activations NHWC in the graph's dtype (bf16 or fp32).
 */
#ifndef HIOS_H
#define HIOS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define HIOS_ABI_VERSION 1

typedef struct hios_graph_s* hios_graph;        /* opaque; caller owns (create/destroy) */
typedef struct hios_schedule_s* hios_schedule;  /* opaque; keeps its graph alive        */

typedef enum {
  HIOS_OK = 0,
  HIOS_E_INVALID = 1,     /* bad argument / malformed graph                 */
  HIOS_E_CYCLE = 2,       /* G has a cycle, or a schedule deadlocks          */
  HIOS_E_SHAPE = 3,       /* shape inference failed / channel mismatch       */
  HIOS_E_OOM = 4,         /* device or host allocation failed                */
  HIOS_E_CUDA = 5,        /* a CUDA runtime/driver call failed               */
  HIOS_E_NCCL = 6,        /* reserved: NCCL fallback transport               */
  HIOS_E_UNSUPPORTED = 7, /* valid request this build cannot execute         */
  HIOS_E_STATE = 8        /* call out of order (e.g. missing costs)          */
} hios_status;

typedef enum { HIOS_F32 = 0, HIOS_BF16 = 1 } hios_dtype;

/* Operator kinds ("convolution, pooling, and linear operators"; the
 * op granularity is SURVEY §8(c) C20: conv + folded BN + ReLU = one op). */
typedef enum {
  HIOS_OP_INPUT = 0,    /* placeholder for the network input (t = its staging)   */
  HIOS_OP_CONV = 1,     /* conv k x k / 1 x n, stride, pad, dilation; scale/shift/ReLU epilogue */
  HIOS_OP_SEPCONV = 2,  /* [weighted sum of inputs] -> reps x (ReLU? -> depthwise -> 1x1 -> scale/shift) -> ReLU? */
  HIOS_OP_MAXPOOL = 3,
  HIOS_OP_AVGPOOL = 4,
  HIOS_OP_GAP = 5,      /* global average pool -> C x 1 x 1                     */
  HIOS_OP_CONCAT = 6,   /* channel concat in input-slot order                    */
  HIOS_OP_ADD = 7,      /* sum_i agg_i x_i, optional ReLU                         */
  HIOS_OP_LINEAR = 8,   /* y = W x + b on the flattened input                     */
  HIOS_OP_IDENTITY = 9
} hios_op_kind;

/* One vertex of G.  Weight layouts (fp32, copied at create):
 *   CONV     weight [out_c][in_c][kh][kw]; scale/shift [out_c] (folded BN;
 *            NULL = 1 / 0); y = relu?(scale * conv(pre_relu ? relu(x) : x, W) + shift)
 *   SEPCONV  weight = concat over r < reps of { dw [c_r][kh][kw], pw [out_c][c_r] }
 *            with c_0 = in_c, c_r = out_c for r > 0; scale/shift [reps][out_c];
 *            stride (sh, sw) on r = 0 only; pad (ph, pw); pre_relu before each
 *            depthwise; relu after the last repetition; agg = input weights
 *            (NULL: exactly one input)
 *   LINEAR   weight [out_c][in_c]; shift = bias [out_c] (NULL = 0)
 *   ADD      agg [n_inputs] (NULL = all 1); relu
 *   MAXPOOL / AVGPOOL  kh, kw, sh, sw, ph, pw, ceil_mode, count_include_pad
 * Output size: floor((H + 2ph - dh(kh-1) - 1)/sh) + 1 (ceil_mode: ceil, and
 * the last window must start inside the input or the left padding). */
typedef struct {
  int32_t kind;
  int32_t in_c, out_c;
  int32_t kh, kw, sh, sw, ph, pw, dh, dw;
  int32_t relu, pre_relu, ceil_mode, count_include_pad, reps;
  const float* weight;
  const float* scale;
  const float* shift;
  const float* agg;
  int64_t cost_ns; /* injected t(v) (host-only scheduling); < 0 = unknown */
} hios_op;

/* One edge (u, v) of G: the output tensor of src is input number `slot` of dst. */
typedef struct {
  int32_t src, dst, slot, reserved;
  int64_t cost_ns; /* injected t(u, v); < 0 = unknown */
} hios_edge;

/* ---------------------------------------------------------------- graph */

/* Build G.  Validates: op kinds and parameters, slot numbering 0..n_in-1 per
 * op, no self loops, acyclicity (HIOS_E_CYCLE), channel/shape consistency
 * (HIOS_E_SHAPE), exactly one HIOS_OP_INPUT with no inputs whose channel count
 * is in_c.  Infers every op's output shape from (in_c, in_h, in_w).  dtype
 * selects the device arithmetic: HIOS_BF16 (tcgen05 tensor cores, fp32
 * accumulate) or HIOS_F32 (CUDA cores). */
hios_status hios_graph_create(const hios_op* ops, int32_t n_ops, const hios_edge* edges,
                              int32_t n_edges, int32_t in_c, int32_t in_h, int32_t in_w,
                              hios_dtype dtype, hios_graph* out);
void hios_graph_destroy(hios_graph g);

/* Inferred output shape (C, H, W) of op `op`. */
hios_status hios_graph_shape(hios_graph g, int32_t op, int32_t* c, int32_t* h, int32_t* w);

/* Cost injection (host-only use, tests, re-use of saved profiles). */
hios_status hios_set_op_cost(hios_graph g, int32_t op, int64_t ns);
hios_status hios_set_edge_cost(hios_graph g, int32_t edge, int64_t ns);
/* t(S) for the set of `n` >= 2 ops (order irrelevant). */
hios_status hios_set_group_cost(hios_graph g, const int32_t* ops, int32_t n, int64_t ns);
/* Fallback t(S) for sets without a table entry or a profiler:
 * t(S) = max(max_v t(v), floor(sum_v t(v) * num / den)).
 * num = 0 disables the model (missing t(S) is then HIOS_E_STATE). */
hios_status hios_set_group_model(hios_graph g, int32_t num, int32_t den);
/* Read back t(v) [n_ops] and t(u, v) [n_edges] (either may be NULL). */
hios_status hios_get_costs(hios_graph g, int64_t* op_ns, int64_t* edge_ns);

/* t(S) of the stage S = ops[0..n) as the scheduler sees it ("t(S)"; the
 * profiling step of P:322): n = 1 -> t(v); else a value injected by
 * hios_set_group_cost, else -- after hios_profile -- the concurrent time of
 * the ops forked onto n streams of devices[0] and joined (measured once,
 * memoised; n <= 8), else the group model.  ops are op ids (any order, no
 * duplicates; the caller states they are independent -- not checked).
 * Writes *ns.  Errors: HIOS_E_INVALID, HIOS_E_STATE (no way to know t(S)),
 * HIOS_E_UNSUPPORTED (n > 8 when measuring), HIOS_E_CUDA. */
hios_status hios_group_cost(hios_graph g, const int32_t* ops, int32_t n, int64_t* ns);

/* ------------------------------------------------------------- profile */

/* Measure t(v) for every op (median of `reps` CUDA-event timings of the op's
 * kernels alone on devices[0]) and t(u, v) for every edge (the incremental
 * cost of delivering u's output to another GPU: a peer store from devices[0]
 * into devices[1] if n_devices >= 2, else into a second buffer on devices[0]).
 * Overwrites injected costs.  Afterwards the scheduler measures t(S) of the
 * candidate groups it needs on devices[0] (lazily, memoised).
 * Errors: HIOS_E_CUDA, HIOS_E_OOM. */
hios_status hios_profile(hios_graph g, const int32_t* devices, int32_t n_devices, int32_t reps);

/* ------------------------------------------------------------ schedule */

/* HIOS-LP (Alg. 1 + Alg. 2) for `n_gpus` >= 1 GPUs and window w >= 1 (the
 * maximum stage size, K = L = w).  Special cases from the same
 * call: n_gpus = 1, window = 1 -> sequential schedule; window = 1 ->
 * "LP-based inter-GPU" only; n_gpus = 1, window = w -> the IOS-style
 * single-GPU stand-in.  Needs t(v), t(u, v) and t(S) (profiled, injected or
 * the group model); otherwise HIOS_E_STATE.  Host-only unless the profiler
 * measures t(S). */
hios_status hios_schedule_lp(hios_graph g, int32_t n_gpus, int32_t window, hios_schedule* out);

/* HIOS-MR, the paper's second scheduler (Alg. 3):
 * mapping-recording DP over the ops in priority order (an n x M table of
 * earliest finish times with back-pointers to the GPU of the previous op),
 * back-tracked from the best GPU of the last op, then Alg. 2.  The extracted
 * pseudo-code is garbled; the reconstruction is SURVEY C17 / DESIGN.md §3.
 * Same arguments, costs and errors as hios_schedule_lp; window = 1 gives
 * "MR-based inter-GPU" only. */
hios_status hios_schedule_mr(hios_graph g, int32_t n_gpus, int32_t window, hios_schedule* out);

/* IOS, the paper's single-GPU comparator (P:158, P:254, P:316 -- "an exact
 * algorithm for the optimal schedule in a single GPU", dynamic programming):
 * on one GPU, the sequence of stages of <= window pairwise-independent ops
 * minimising L = sum t(S).  Exact DP over finished-op sets, decomposed at cut
 * vertices (ops comparable with every other op); a block of more than 32 ops
 * is cut into topological-order chunks (as IOS partitions large graphs; exact
 * per chunk -- Inception-v3, SqueezeNet, RandWire need no cut).  t(S)
 * as for hios_schedule_lp (measured lazily after hios_profile, injected, or
 * the group model).  max_states bounds the DP (<= 0: 2^22).  Writes *out
 * (caller owns).  Errors: HIOS_E_INVALID, HIOS_E_STATE, HIOS_E_UNSUPPORTED
 * (state budget exceeded), HIOS_E_CUDA. */
hios_status hios_schedule_ios(hios_graph g, int32_t window, int64_t max_states, hios_schedule* out);

/* Import a schedule: op_gpu[v] in [0, n_gpus), op_stage[v] = stage index on
 * that GPU (stages numbered 0..K_i-1; ops sharing an index form one stage).
 * Checked for feasibility (C6): HIOS_E_INVALID (dependent ops in a stage,
 * stage larger than `window`), HIOS_E_CYCLE (deadlock). */
hios_status hios_schedule_import(hios_graph g, int32_t n_gpus, int32_t window,
                                 const int32_t* op_gpu, const int32_t* op_stage,
                                 hios_schedule* out);
void hios_schedule_destroy(hios_schedule s);

/* Predicted latency L of Q under the cost model. */
hios_status hios_schedule_latency_ns(hios_schedule s, int64_t* predicted);
/* Q as per-op (gpu, stage index); n_stages[g] for g < n_gpus (any may be NULL). */
hios_status hios_schedule_stages(hios_schedule s, int32_t* op_gpu, int32_t* op_stage,
                                 int32_t* n_stages);

/* ----------------------------------------------------------------- run */

/* Placement of the schedule's logical GPUs: devices[i] = CUDA device of
 * logical GPU i (several logical GPUs may share one device: they then run on
 * separate streams of it).  Default: logical GPU i -> device i % n_visible.
 * Must precede the first run. */
hios_status hios_schedule_place(hios_schedule s, const int32_t* devices, int32_t n);

/* Transport of the cross-GPU edges; must precede the
 * first run.
 *   HIOS_TRANSPORT_PEER (default): the producer's epilogue stores straight into
 *     every consumer GPU's buffer (peer memory over NVLink / CUDA IPC), then a
 *     system-scope release of an epoch flag; the consumer stage waits on the
 *     flag device-side.
 *   HIOS_TRANSPORT_COPY: the producer writes locally; a copy-engine transfer
 *     (cudaMemcpy2DAsync) into the consumer's buffer follows it, then the flag
 *     -- the paper's launch-after-transfer design (CUDA-aware MPI).
 *   HIOS_TRANSPORT_NCCL: the producer writes locally; ncclSend / ncclRecv on a
 *     per-GPU communication stream in one global transfer order (the stage
 *     DAG's topological order), the consumer stage waits for the receive --
 *     the fallback baseline P:318 names.  Needs one process per GPU
 *     (hios_schedule_bind_rank) and hios_schedule_nccl_init; edges between
 *     logical GPUs of the same process use the copy transport.
 * Errors: HIOS_E_INVALID (unknown transport), HIOS_E_STATE (already run). */
typedef enum { HIOS_TRANSPORT_PEER = 0, HIOS_TRANSPORT_COPY = 1, HIOS_TRANSPORT_NCCL = 2 } hios_transport;
hios_status hios_schedule_transport(hios_schedule s, int32_t transport);

/* How a stage's concurrent group is launched; must
 * precede the first run.
 *   HIOS_STAGE_STREAMS (default): every op of the stage on its own stream of
 *     the GPU (fork from / join into the stage's first stream), each kernel
 *     free to take any SM the hardware gives it.
 *   HIOS_STAGE_GROUPED: the stage's plain tcgen05 convolutions as ONE
 *     persistent launch (conv_tc_group_kernel) that partitions the SMs across
 *     them -- op i owns a CTA range sized to minimise the stage's makespan from
 *     the measured t(v) -- and the stage's other ops on forked streams.
 *     (hios_profile measures t(S) with streams.)  (Measured on one B200,
 *     Inception-v3 HIOS-LP w = 5: 0.80 ms grouped vs 0.74 ms streams at 1024^2;
 *     DESIGN.md §6.)
 *   HIOS_STAGE_DATAFLOW: the stages' ops in the schedule's order, op i of a
 *     stage on stream i of its GPU, each waiting only for its own inputs and
 *     the previous op of its stream instead of the whole previous stage (the
 *     stage boundary join of P:86 relaxed to the data dependencies; at
 *     most |S| <= w ops in flight per GPU as in the stage model).
 *   HIOS_STAGE_AUTO: both STREAMS and DATAFLOW graphs are captured; the first
 *     run (its results are STREAMS') then replays each 9 times and keeps the
 *     faster (median wall time of launch + synchronize) for every later run --
 *     measured selection, like the profiler's t(S).  One process
 *     driving all its logical GPUs only (otherwise STREAMS).
 * Errors: HIOS_E_INVALID (unknown mode), HIOS_E_STATE (already run). */
typedef enum {
  HIOS_STAGE_STREAMS = 0,
  HIOS_STAGE_GROUPED = 1,
  HIOS_STAGE_DATAFLOW = 2,
  HIOS_STAGE_AUTO = 3
} hios_stage_mode;
hios_status hios_schedule_stage_mode(hios_schedule s, int32_t mode);
/* The stage mode the schedule's graphs execute (after the first run; AUTO
 * resolves to STREAMS or DATAFLOW).  Errors: HIOS_E_INVALID, HIOS_E_STATE
 * (not run yet). */
hios_status hios_schedule_stage_mode_used(hios_schedule s, int32_t* mode);

/* NCCL transport set-up.  hios_nccl_unique_id writes a 128-byte ncclUniqueId
 * (call on one rank, broadcast the bytes); hios_schedule_nccl_init creates
 * this rank's communicator (nranks processes, this one = rank, on the device
 * of its logical GPUs) after hios_schedule_bind_rank.  libnccl.so.2 is
 * loaded at run time (HIOS_NCCL_LIB overrides the path).  Errors: HIOS_E_NCCL
 * (library missing, init failed), HIOS_E_UNSUPPORTED (this rank owns logical
 * GPUs on several devices), HIOS_E_STATE (not in rank mode). */
hios_status hios_nccl_unique_id(void* id128);
hios_status hios_schedule_nccl_init(hios_schedule s, const void* id128, int32_t nranks, int32_t rank);

/* The global order of the cross-GPU transfers (one per (producer op,
 * consumer logical GPU) pair) the NCCL transport posts its sends / receives
 * in: ascending position of the producer's stage in a topological order of the
 * stage DAG (data edges + per-GPU stage order), ties by producer id, then
 * consumer GPU.  src_op / dst_gpu [cap] (caller-owned), *n = count (if the
 * arrays are NULL only *n is written). */
hios_status hios_schedule_transfers(hios_schedule s, int32_t* src_op, int32_t* dst_gpu, int32_t cap, int32_t* n);

/* Multi-process execution (one process per GPU): this process executes only
 * the logical GPUs i with owner[i] == rank (all of them placed on one device;
 * hios_ipc_import rejects a rank spanning several devices, HIOS_E_UNSUPPORTED).  Cross-process edges use CUDA IPC
 * peer memory: after hios_ipc_export on every rank, each rank imports every
 * other rank's blob.  blob is caller-owned; *len in: capacity, out: size. */
hios_status hios_schedule_bind_rank(hios_schedule s, const int32_t* owner, int32_t n, int32_t rank);
hios_status hios_ipc_export(hios_schedule s, void* blob, size_t* len);
hios_status hios_ipc_import(hios_schedule s, int32_t rank, const void* blob, size_t len);

/* Number of fp32 elements of the network output (the unique sink op's C*H*W). */
hios_status hios_output_numel(hios_schedule s, int64_t* n);

/* Run one batch-1 inference under Q.  `input` = fp32 NCHW host array
 * (in_c*in_h*in_w), `output` = fp32 NCHW host array (hios_output_numel).
 * The first call lowers Q (buffers, concat slices, peer pointers, streams,
 * flags) and captures one CUDA graph per logical GPU; every call then copies
 * the input to the INPUT op's GPU, launches all graphs, waits, and copies the
 * sink's output back.  In rank mode, input/output may be NULL on ranks that do
 * not own the INPUT / sink op.  Not reentrant per schedule. */
hios_status hios_run(hios_schedule s, const float* input, float* output);

/* Same with device pointers: d_in = fp32 NCHW on the INPUT op's device,
 * d_out = fp32 NCHW on the sink op's device; `stream` (cudaStream_t, may be
 * NULL) orders the run after prior work on it and later work after the run. */
hios_status hios_run_device(hios_schedule s, const void* d_in, void* d_out, void* stream);

/* After a run: fp32 NCHW copy of op `op`'s output (C*H*W elements) read from
 * its GPU (debug / per-op parity). */
hios_status hios_read_op_output(hios_schedule s, int32_t op, float* host, int64_t n);

/* Per-op device time of the last hios_run_timed call (ns, [n_ops]; ops not run
 * locally are -1).  hios_run_timed = hios_run_device with an instrumented
 * graph (CUDA events around each op; stages still run concurrently). */
hios_status hios_run_timed(hios_schedule s, const void* d_in, void* d_out, void* stream,
                           int64_t* op_ns);

/* Uninstrumented device time of each op's kernels as configured in Q (the
 * stage context decides the conv tile plan), each op timed alone on its
 * logical GPU's device: per rep the L2 is flushed by writing `flush_bytes`
 * (0 = no flush), then CUDA events recorded as graph nodes on the launching
 * stream bracket the op's kernels only; median of `reps` (>= 1) after one
 * warm-up.  Lowers/captures Q first if needed.  op_ns [n_ops] (caller-owned):
 * ns, or -1 for ops not executed by this process, the INPUT placeholder and
 * concats (zero-copy).  Errors: HIOS_E_INVALID, HIOS_E_CUDA, HIOS_E_OOM. */
hios_status hios_time_ops(hios_schedule s, int32_t reps, int64_t flush_bytes, int64_t* op_ns);

/* Number of kernels one run launches on this process's GPUs (graph nodes
 * that are kernels written in this library). */
hios_status hios_kernel_count(hios_schedule s, int64_t* n);

/* Tile plan of op `op`'s tcgen05 convolution as lowered for Q ("the
 * convolution ... operators"), for inspection and tests:
 * solo = 0 the plan used inside its stage, 1 the plan used when the op runs
 * alone (a singleton stage, t(v) profiling).  plan[8] (caller-owned) =
 * {A-operand mode: 1 tap, 2 halo, 3 virtual-grid halo; N tile; output tiles;
 * epilogue: 0 smem staging, 1 TMA bulk-tensor stores, 2 direct stores;
 * 1 = 256-bit direct stores; output rows per tile; pipeline stages;
 * K-steps per stage}; all zero for ops without a tcgen05
 * conv (other kinds, fp32 graphs, CUDA-core stems).  Errors: HIOS_E_INVALID
 * (NULL, op out of range), HIOS_E_STATE (Q not run yet). */
hios_status hios_op_plan(hios_schedule s, int32_t op, int32_t solo, int32_t* plan);

/* *relu = 1 when op `op`'s stored output (hios_read_op_output) is ReLU(y)
 * rather than y: every consumer applies ReLU to it first (pre-ReLU convs,
 * single-input separable convs and ReLU adds, or a concat whose consumers all
 * do -- NASNet's ReLU -> conv -> BN cell inputs), so the executor applies the
 * ReLU in the producer's epilogue instead of making a ReLU'd copy for the
 * consumers; the network output never is.  Errors: HIOS_E_INVALID,
 * HIOS_E_STATE (not run yet). */
hios_status hios_op_output_relu(hios_schedule s, int32_t op, int32_t* relu);

/* ------------------------------------------------------------------ misc */
const char* hios_last_error(void);
int32_t hios_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* HIOS_H */
