#!/usr/bin/env python
"""bench.py -- batch-1 DAG-CNN inference latency under an HIOS-LP schedule on
N B200 GPUs (BASELINE.json metric), through the C-ABI (libhios.so).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--model inception_v3]
                  [--size 1024] [--window 3] [--dtype bf16] [--impl reference]

One step = one inference of the workload (configs[1]: Inception-v3, batch 1,
1x3x1024x1024 synthetic input, random-init weights) with the whole hot path:
input layout conversion -> every operator kernel of every stage on every GPU
(cross-GPU edges as peer stores + device-side flags) -> output conversion.
Profiling (t(v), t(u,v), t(S)) and HIOS-LP scheduling run once before the
timed region; their wall time is reported (the paper's "time cost of
scheduling optimization").

Timing: W untimed warm-up steps; then K steps, each preceded by an L2 flush
(a 256 MiB write, outside the events) and bracketed by CUDA events on the
launching stream; barrier + synchronize on both sides; max over ranks.
`e2e` = the same latency through hios_run with pinned host buffers (H2D of the
fp32 input and D2H of the logits inside the timed region, host wall clock).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "batch-1 DAG-CNN inference latency (ms) at 1/2/4/8 B200 vs critical-path roofline"


def peaks():
    p = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "src": "fallback"}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            m = json.load(f)
        p.update({k: m[k] for k in ("hbm_gbs", "bf16_tflops", "bf16_tflops_sustained") if k in m})
        p["src"] = "measured"
    except Exception:
        pass
    p["nvlink_gbs"] = 770.0  # measured peer copy per direction (B200_PROFILING.md)
    # FP32 CUDA-core peak (the fp32 path's roofline): measured by tools/fp32_peak.cu
    # on this pool's B200 (profiles/fp32_peak.json), else 148 SMs x 128 lanes x 2 x 1.965 GHz
    p["fp32_tflops"], p["fp32_src"] = 74.45, "nominal (148 x 128 FFMA lanes x 2 x 1.965 GHz)"
    try:
        with open(os.path.join(ROOT, "profiles", "fp32_peak.json")) as f:
            p["fp32_tflops"] = float(json.load(f)["fp32_tflops"])
            p["fp32_src"] = "measured (tools/fp32_peak.cu, profiles/fp32_peak.json)"
    except Exception:
        pass
    return p


def compute_peak(pk, dtype):
    """Dense-contraction peak for the path's arithmetic (TFLOP/s): tcgen05 bf16
    burst for bf16, the FP32 CUDA-core peak for fp32."""
    return pk["bf16_tflops"] if dtype == "bf16" else pk["fp32_tflops"]


# the paper's own relative results (§VI-D/E), quoted with its hardware;
# context for speedup_vs_*, not a target (different GPUs, interconnect, sizes)
PAPER_NUMBERS = {
    "hardware": "2x NVIDIA A40 (48 GB GDDR6, 696 GB/s), one NVLink bridge 112.5 GB/s bidirectional; "
                "cuDNN 8.8.1 engine of IOS + CUDA-aware MPI (P:286-290)",
    "timing": "mean of 36 runs (P:290)",
    "hios_lp_vs_sequential": "6.1%-19.7% lower latency on Inception-v3, up to 14.5% on NASNet (P:308)",
    "hios_lp_vs_ios": "3.3%-16.5% lower on Inception-v3, up to 11.1% on NASNet (P:308); "
                      "5.4% HIGHER than IOS on NASNet at the small input (P:316)",
    "hios_lp_vs_hios_mr": "10.9%-16.8% lower on Inception-v3, 8.8%-16.2% on NASNet (P:310)",
    "reduction_ratio_vs_ios": "HIOS-LP's latency reduction over sequential is 9.9x (large input) and 4.5x "
                              "(small) IOS's for Inception-v3, 3.8x for NASNet large (P:316)",
    "inter_gpu_share": "LP inter-GPU mapping gives 98.2% (large) / 81.6% (small) of HIOS-LP's reduction on "
                       "Inception-v3, ~100% on NASNet (P:318)",
}


# ------------------------------------------------------------ op accounting
def op_work(g, shapes, esz):
    """Algorithmic FLOPs and HBM bytes per op (SURVEY §8(d) units): conv
    F = 2 K (C/g) R S P Q, B = (C H W + K C R S + K P Q) elt; pools / add / gap
    read their inputs and write their output once; concat is 0 bytes when
    producers write in place (the executor copies only misaligned slices)."""
    F = np.zeros(g.n_ops)
    B = np.zeros(g.n_ops)
    preds = {o.id: g.preds(o.id) for o in g.ops}
    for o in g.ops:
        C, P, Q = shapes[o.id]
        ins = [shapes[u] for u in preds[o.id]]
        inb = sum(c * h * w for (c, h, w) in ins) * esz
        outb = C * P * Q * esz
        if o.kind == "conv":
            ci, hi, wi = ins[0]
            F[o.id] = 2.0 * o.out_c * ci * o.kh * o.kw * P * Q
            B[o.id] = inb + o.out_c * ci * o.kh * o.kw * esz + outb
        elif o.kind == "sepconv":
            ci = ins[0][0]
            f = b = 0.0
            for r in range(o.reps):
                c = ci if r == 0 else o.out_c
                f += 2.0 * c * o.kh * o.kw * P * Q + 2.0 * o.out_c * c * P * Q
                b += (c * o.kh * o.kw + o.out_c * c) * esz + 2 * c * P * Q * esz
            F[o.id] = f
            B[o.id] = b + inb + outb
        elif o.kind == "linear":
            F[o.id] = 2.0 * o.out_c * o.in_c
            B[o.id] = (o.out_c * o.in_c) * esz + inb + outb
        elif o.kind in ("maxpool", "avgpool", "add", "gap", "identity"):
            B[o.id] = inb + outb
        elif o.kind == "concat":
            B[o.id] = 0.0
        elif o.kind == "input":
            B[o.id] = C * P * Q * 4 + outb  # fp32 NCHW read + NHWC write
    return F, B


def critical_path_bound(g, F, B, op_gpu, op_stage, n_gpus, pk, esz, shapes, dtype="bf16"):
    """Schedule critical-path lower bound: stage roof =
    max(max_v roof(v), sum F / Pi, sum B / beta); stages on a GPU serialise;
    cross-GPU edges cost bytes / NVLink (overlap form: an edge may start when
    its producer starts, so it adds max(0, t_edge - roof(u))).  Returns s."""
    Pi = compute_peak(pk, dtype) * 1e12
    beta = pk["hbm_gbs"] * 1e9
    nvl = pk["nvlink_gbs"] * 1e9
    roof = np.maximum(F / Pi, B / beta)
    stages = {}
    for v in range(g.n_ops):
        stages.setdefault((int(op_gpu[v]), int(op_stage[v])), []).append(v)
    cost = {k: max(max(roof[v] for v in S), sum(F[v] for v in S) / Pi, sum(B[v] for v in S) / beta)
            for k, S in stages.items()}
    where = {v: (int(op_gpu[v]), int(op_stage[v])) for v in range(g.n_ops)}
    preds = {k: [] for k in stages}
    for k in stages:
        if k[1] > 0:
            preds[k].append(((k[0], k[1] - 1), 0.0))
    for (u, v, _) in g.edges:
        su, sv = where[u], where[v]
        if su[0] != sv[0]:
            c, h, w = shapes[u]
            t = c * h * w * esz / nvl
            preds[sv].append((su, max(0.0, t - roof[u])))
        else:
            preds[sv].append((su, 0.0))
    fin = {}

    def finish(k):
        if k not in fin:
            st = max([finish(p) + d for (p, d) in preds[k]] or [0.0])
            fin[k] = st + cost[k]
        return fin[k]

    sys.setrecursionlimit(100000)
    return max(finish(k) for k in stages)


# ------------------------------------------------------------ clocks
class Clocks:
    """SM clock + throttle reasons sampled DURING the timed region.

    A thread polls NVML every ~2 ms (the timed region of a 1 ms inference is
    only tens of ms, far below nvidia-smi's sampling period); ctypes releases
    the GIL while the main thread launches, so sampling does not perturb it.
    Falls back to `nvidia-smi -lms` if NVML is unavailable."""

    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, idx):
        self.sm, self.mx, self.reasons, self.err = [], [], set(), None
        self.stop_ev = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            try:
                import torch
                nidx = torch.cuda._get_nvml_device_index(idx)
            except Exception:
                nidx = idx
            hd = pynvml.nvmlDeviceGetHandleByIndex(nidx)
            bits = {"hw_slowdown": pynvml.nvmlClocksEventReasonHwSlowdown,
                    "hw_thermal_slowdown": pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                    "sw_thermal_slowdown": pynvml.nvmlClocksEventReasonSwThermalSlowdown,
                    "sw_power_cap": pynvml.nvmlClocksEventReasonSwPowerCap}
            self.mx.append(float(pynvml.nvmlDeviceGetMaxClockInfo(hd, pynvml.NVML_CLOCK_SM)))

            def sample():
                self.sm.append(float(pynvml.nvmlDeviceGetClockInfo(hd, pynvml.NVML_CLOCK_SM)))
                r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(hd)
                for n, bit in bits.items():
                    if r & bit:
                        self.reasons.add(n)

            def loop():
                while not self.stop_ev.is_set():
                    try:
                        sample()
                    except Exception as e:  # noqa: BLE001
                        self.err = str(e)
                        return
                    time.sleep(0.002)

            self.t = threading.Thread(target=loop, daemon=True)
            self.t.start()
        except Exception as e:  # noqa: BLE001
            self.t = None
            self.err = f"nvml unavailable: {e}"

    def stop(self):
        self.stop_ev.set()
        if self.t is not None:
            self.t.join()
        out = {"sm_mhz": float(np.median(self.sm)) if self.sm else None,
               "sm_max_mhz": float(max(self.mx)) if self.mx else None,
               "samples": len(self.sm), "reasons": sorted(self.reasons), "source": "nvml, 2 ms poll"}
        if self.err:
            out["error"] = self.err
        return out


# ------------------------------------------------------------ CPU oracle leg
def _oracle_walk(g, W, x, upto=None):
    """The oracle as it stands (oracle/infer.py run_op, in topological order,
    fp64 numpy), op by op with per-op wall times; values dropped after their
    last consumer.  `upto`: stop after that many non-input ops (a sample).
    Returns (seconds, per-op seconds {id: s}, ops run).  Shapes come from the
    oracle itself -- nothing of the product is imported."""
    from oracle import infer
    preds = {o.id: g.preds(o.id) for o in g.ops}
    left = {o.id: 0 for o in g.ops}
    for (u, _, _) in g.edges:
        left[u] += 1
    vals, per, k = {}, {}, 0
    t0 = time.perf_counter()
    for o in g.ops:
        if upto is not None and o.kind != "input" and k >= upto:
            break
        a = time.perf_counter()
        if o.kind == "input":
            vals[o.id] = x[0].astype(np.float64)
        else:
            vals[o.id] = infer.run_op(o, [vals[u] for u in preds[o.id]], W[o.id])
            k += 1
        for u in preds[o.id]:
            left[u] -= 1
            if left[u] == 0:
                vals.pop(u, None)
        per[o.id] = time.perf_counter() - a
    return time.perf_counter() - t0, per, k


def oracle_leg(g, W, x, n_runs, budget_s):
    """Time the fp64 CPU oracle on the host cores for n_runs steps within
    ~budget_s of CPU work.  The first pass is a whole inference (per-op times,
    untimed warm-up).  If n_runs whole inferences fit the budget, every step is
    a whole inference (no extrapolation).  Otherwise every step runs the same
    prefix of operators in topological order (the sample) and is scaled by that
    prefix's MEASURED share of the whole warm-up inference.
    Returns (list of per-step ms per inference, sample description, threads)."""
    t_full, per, n_all = _oracle_walk(g, W, x)
    threads = _blas_threads()
    if t_full * n_runs <= budget_s:
        vals = []
        for _ in range(n_runs):
            t, _, _ = _oracle_walk(g, W, x)
            vals.append(t * 1e3)
        return vals, (f"whole inference of {g.name} ({n_all} ops), fp64 numpy oracle "
                      f"(oracle/infer.py), {n_runs} runs"), threads
    per_step = budget_s / max(n_runs, 1)
    acc, upto = 0.0, 0
    for o in g.ops:
        if o.kind == "input":
            acc += per[o.id]
            continue
        if acc + per[o.id] > per_step and upto > 0:
            break
        acc += per[o.id]
        upto += 1
    vals = []
    for _ in range(n_runs):
        t, _, k = _oracle_walk(g, W, x, upto)
        vals.append(t / (acc / t_full) * 1e3)
    return vals, (f"first {upto} of {n_all} ops of {g.name} in topological order per step "
                  f"({100 * acc / t_full:.1f}% of a whole inference's measured oracle time, "
                  f"whole inference {t_full:.1f} s), scaled by that measured share; fp64 numpy oracle"), threads


def _blas_threads():
    try:
        from threadpoolctl import threadpool_info
        n = [i.get("num_threads", 0) for i in threadpool_info() if i.get("user_api") == "blas"]
        if n:
            return int(max(n))
    except Exception:
        pass
    return len(os.sched_getaffinity(0))


# ------------------------------------------------------------ N > 1 plumbing
def owners(M, world):
    """Logical GPU i of the schedule is executed by rank i % world (one
    process per GPU; HIOS-LP may leave some GPUs idle, P:82 'm <= M')."""
    return [i % world for i in range(M)]


def share_schedule(h, dist, G, g, S, M, window, rank):
    """Rank 0 profiled and scheduled; every other rank receives t(v), t(u,v)
    and Q (per-op GPU + stage) and imports the identical schedule."""
    if rank == 0:
        opc, edc = h.hios_get_costs(G)
        og, ost, _ = h.hios_schedule_stages(S)
        obj = [opc.tolist(), edc.tolist(), og.tolist(), ost.tolist()]
    else:
        obj = [None, None, None, None]
    dist.broadcast_object_list(obj, src=0)
    opc, edc, og, ost = obj
    if rank != 0:
        for v in range(g.n_ops):
            h.hios_set_op_cost(G, v, int(opc[v]))
        for e in range(g.n_edges):
            h.hios_set_edge_cost(G, e, int(edc[e]))
        h.hios_set_group_model(G, 7, 10)  # t(S) of the imported groups (prediction only)
        S = h.hios_schedule_import(G, M, window, og, ost)
    return S


def bind_and_exchange(h, dist, S, M, world, rank, dev, transport="peer"):
    """Each rank owns its logical GPUs; device buffers and flag words are
    exported as CUDA IPC handles and mapped by every other rank, so producers
    store straight into consumer buffers (peer memory over NVLink).  With the
    NCCL transport rank 0's ncclUniqueId is broadcast and every rank creates
    its communicator (the IPC maps then only carry same-process flags)."""
    own = owners(M, world)
    h.hios_schedule_place(S, [dev] * M)
    h.hios_schedule_bind_rank(S, own, rank)
    if transport == "nccl":
        uid = [h.hios_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        h.hios_schedule_nccl_init(S, uid[0], world, rank)
    blob = h.hios_ipc_export(S)
    blobs = [None] * world
    dist.all_gather_object(blobs, blob)
    for r in range(world):
        if r != rank:
            h.hios_ipc_import(S, r, blobs[r])
    return own


def max_over_ranks(dist, x, world):
    if world <= 1:
        return x
    import torch
    t = torch.tensor([float(x)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


# ------------------------------------------------------------ workload sweep
def measure_workload(h, torch, model, sz, M, args, dev, stream, flush, pk, dtype):
    """One more BASELINE.json workload (another size or another benchmark DAG)
    in the same run: profile, then HIOS-LP (M, w), sequential (1, 1) and the
    IOS-style stand-in (1, w), each timed like the main line (device events,
    L2 flushed between steps), plus the schedule's critical-path bound."""
    from workloads import gen, graphs
    gs = graphs.build(model, sz)
    Ws = gen.make_weights(gs)
    xs = gen.make_input(gs)
    esz = 2 if dtype == "bf16" else 4
    Gs = h.hios_graph_create(gs.ops, gs.edges, gs.in_c, gs.in_h, gs.in_w, dtype, Ws)
    shp = {o.id: h.hios_graph_shape(Gs, o.id) for o in gs.ops}
    t0 = time.perf_counter()
    h.hios_profile(Gs, [dev], 5)
    row = {"input": f"1x{gs.in_c}x{sz}x{sz}", "dtype": dtype, "ops": gs.n_ops, "deps": gs.n_edges,
           "profile_s": time.perf_counter() - t0}
    din = torch.from_numpy(xs).to(f"cuda:{dev}")
    dout = None
    for name, (m_, w_) in {"hios_lp": (M, args.window), "sequential": (1, 1),
                           "ios_style": (1, args.window), "ios": (1, args.window)}.items():
        t0 = time.perf_counter()
        if name == "ios":
            # exact single-GPU DP, state budget bounded so the lazily
            # profiled t(S) stay within the bench's time (NASNet: see DESIGN)
            try:
                Sx = h.hios_schedule_ios(Gs, w_, args.ios_states)
            except h.HiosError as ex:
                row["ios_unavailable"] = str(ex)
                continue
        else:
            Sx = h.hios_schedule_lp(Gs, m_, w_)
        t_s = time.perf_counter() - t0
        h.hios_schedule_stage_mode(Sx, args.stage_mode)
        if m_ > 1:
            ndev = torch.cuda.device_count()
            h.hios_schedule_place(Sx, [i % ndev for i in range(m_)])
        if dout is None:
            dout = torch.empty(h.hios_output_numel(Sx), dtype=torch.float32, device=f"cuda:{dev}")
        for _ in range(3):
            h.hios_run_device(Sx, din.data_ptr(), dout.data_ptr(), stream.cuda_stream)
        if name == "hios_lp":
            row["stage_mode"] = h.hios_schedule_stage_mode_used(Sx)
        ev = []
        for i in range(max(5, args.steps // 3)):
            flush.fill_(float(i))
            a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a_.record(stream)
            h.hios_run_device(Sx, din.data_ptr(), dout.data_ptr(), stream.cuda_stream)
            b_.record(stream)
            ev.append((a_, b_))
        torch.cuda.synchronize()
        row[name + "_ms"] = float(np.mean([a_.elapsed_time(b_) for a_, b_ in ev]))
        row[name + "_predicted_ms"] = h.hios_schedule_latency_ns(Sx) / 1e6
        if name == "hios_lp":
            og, ost, _ = h.hios_schedule_stages(Sx)
            Fs, Bs = op_work(gs, shp, esz)
            row["cp_bound_ms"] = critical_path_bound(gs, Fs, Bs, og, ost, M, pk, esz, shp, dtype) * 1e3
            row["seq_roofline_ms"] = float(np.maximum(Fs / (compute_peak(pk, dtype) * 1e12),
                                                      Bs / (pk["hbm_gbs"] * 1e9)).sum() * 1e3)
            row["compute_peak_tflops"] = compute_peak(pk, dtype)
            row["gflop"] = float(Fs.sum() / 1e9)
            row["gpus_used"] = int(len(set(og.tolist())))
            row["schedule_s"] = t_s
        del Sx
    row["cp_frac"] = row["cp_bound_ms"] / row["hios_lp_ms"]
    row["speedup_vs_sequential"] = row["sequential_ms"] / row["hios_lp_ms"]
    row["speedup_vs_ios_style"] = row["ios_style_ms"] / row["hios_lp_ms"]
    if "ios_ms" in row:
        row["speedup_vs_ios"] = row["ios_ms"] / row["hios_lp_ms"]
    del Gs
    return row


# ------------------------------------------------------------ main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--model", default="inception_v3")
    ap.add_argument("--size", type=int, default=1024)
    ap.add_argument("--window", type=int, default=5)
    ap.add_argument("--dtype", default="bf16")
    ap.add_argument("--impl", default="hios", choices=["hios", "reference"])
    ap.add_argument("--cpu-budget", type=float, default=30.0,
                    help="seconds of oracle CPU work for the main arm's cpu_baseline")
    ap.add_argument("--ref-budget", type=float, default=200.0,
                    help="seconds of oracle CPU work for the whole --impl reference run")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--sweep", default="2048,4096,randwire_ws@2048,nasnet_a_large@2048,squeezenet@2048,4096:f32",
                    help="extra input sizes timed on 1 GPU (HIOS-LP / sequential / IOS-style), '' to skip")
    ap.add_argument("--transport", default="peer", choices=["peer", "copy", "nccl"],
                    help="cross-GPU edge transport (N > 1): fused peer stores, copy engine, NCCL send/recv")
    ap.add_argument("--stage-mode", default="auto", choices=["streams", "grouped", "dataflow", "auto"],
                    help="stage execution: per-op streams joined per stage, one grouped conv launch per stage "
                         "(f2), per-op input waits (dataflow), or auto (both captured, the faster kept after "
                         "the first run); applied to every schedule the bench times")
    ap.add_argument("--ios-states", type=int, default=1 << 14,
                    help="state budget of the exact IOS DP in the size sweep (its t(S) are profiled lazily: "
                         "NASNet-A 2048^2 needs 2^18, ~5 min)")
    ap.add_argument("--logical", type=int, default=0,
                    help="single process: schedule over this many logical GPUs (aliased on visible devices)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    from workloads import gen, graphs
    g = graphs.build(args.model, args.size)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    workload = f"{args.model}_{args.size}"
    cfg = {"workload": workload, "model": args.model, "global_batch": 1,
           "input": f"1x{g.in_c}x{g.in_h}x{g.in_w}", "ops": g.n_ops, "deps": g.n_edges,
           "window": args.window, "parallelism": f"inter-op x{args.gpus}",
           "l2": "flushed between steps (256 MiB write)", "weights": "random-init (seeded)"}

    if args.impl == "reference":
        # the tier's reference arm: the fp64 CPU oracle as it stands, on the
        # host cores, rank 0 only (other ranks exit without work)
        if rank != 0:
            return 0
        vals, desc, threads = oracle_leg(g, W, x, args.warmup + args.steps, args.ref_budget)
        steps_ms = vals[args.warmup:]
        v = float(np.mean(steps_ms))
        line = {"metric": METRIC, "value": v, "unit": "ms", "n_gpus": args.gpus, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": v, "higher_is_better": False, "scaling": "weak",
                "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
                "config": cfg,
                "cpu_baseline": {"value": v, "unit": "ms", "cores": threads, "kind": "oracle", "sample": desc,
                                 "median": float(np.median(steps_ms))},
                "e2e": {"value": v, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line))
        return 0

    import torch
    import torch.distributed as dist
    from paper_conf_cluster_kundus23_b200 import hios as h

    ndev_vis = torch.cuda.device_count()
    dev = local_rank % ndev_vis
    torch.cuda.set_device(dev)
    if world > 1:
        # host-side plumbing only (costs, schedule, IPC handles, barriers,
        # max-over-ranks timing): activations never go through a collective
        dist.init_process_group(os.environ.get("HIOS_DIST_BACKEND", "gloo"))
    esz = 2 if args.dtype == "bf16" else 4
    pk = peaks()
    M = args.gpus if world > 1 else max(args.gpus, args.logical or 1)

    # ---------------- graph, profile, schedules
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, args.dtype, W)
    shapes = {o.id: h.hios_graph_shape(G, o.id) for o in g.ops}
    t0 = time.perf_counter()
    if rank == 0:
        h.hios_profile(G, [dev] + ([(dev + 1) % ndev_vis] if ndev_vis > 1 else []), 10)
    t_prof = time.perf_counter() - t0
    t0 = time.perf_counter()
    S = h.hios_schedule_lp(G, M, args.window) if rank == 0 else None
    t_sched = time.perf_counter() - t0
    if world > 1:
        S = share_schedule(h, dist, G, g, S, M, args.window, rank)
    h.hios_schedule_transport(S, args.transport)
    h.hios_schedule_stage_mode(S, args.stage_mode)
    cfg["transport"], cfg["stage_mode"] = args.transport, args.stage_mode
    if world > 1:
        bind_and_exchange(h, dist, S, M, world, rank, dev, transport=args.transport)
    elif M > 1:
        ndev = torch.cuda.device_count()
        h.hios_schedule_place(S, [i % ndev for i in range(M)])
    op_gpu, op_stage, n_stages = h.hios_schedule_stages(S)
    predicted_ms = h.hios_schedule_latency_ns(S) / 1e6

    stream = torch.cuda.current_stream()
    d_in = torch.from_numpy(x).to(f"cuda:{dev}")
    n_out = h.hios_output_numel(S)
    d_out = torch.empty(n_out, dtype=torch.float32, device=f"cuda:{dev}")
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=f"cuda:{dev}")

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def run_dev(s):
        h.hios_run_device(s, d_in.data_ptr(), d_out.data_ptr(), stream.cuda_stream)

    def timed_loop(s, steps, timed_fn=None):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(steps)]
        for i in range(steps):
            flush.fill_(float(i))
            ev[i][0].record(stream)
            run_dev(s) if timed_fn is None else timed_fn(s)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
        return [a.elapsed_time(b) for (a, b) in ev]

    for _ in range(args.warmup):
        run_dev(S)
    barrier()
    if args.stage_mode == "auto":
        cfg["stage_mode"] = "auto->" + h.hios_schedule_stage_mode_used(S)
    clk = Clocks(dev)
    barrier()
    ncu = bool(os.environ.get("HIOS_NCU"))
    if ncu:
        torch.cuda.profiler.start()
    wall0 = time.perf_counter()
    times = timed_loop(S, args.steps)
    barrier()
    if ncu:
        torch.cuda.profiler.stop()
    wall = time.perf_counter() - wall0
    clocks = clk.stop()
    total = max_over_ranks(dist, float(np.sum(times)), world)
    ms = total / args.steps

    # ---------------- end-to-end through hios_run (pinned host buffers)
    xin = torch.from_numpy(x).pin_memory().numpy() if True else x
    e2e = []
    for i in range(args.warmup + args.steps):
        flush.fill_(float(i))
        barrier()
        t0 = time.perf_counter()
        y = h.hios_run(S, xin if (world == 1 or int(op_gpu[0]) % world == rank or True) else None)
        e2e.append((time.perf_counter() - t0) * 1e3)
    # median: host-side copies see occasional OS / PCIe stalls (measured: the
    # mean moved 1.06 -> 1.58 ms between two boxes with the same device time)
    e2e_ms = max_over_ranks(dist, float(np.median(e2e[args.warmup:])), world)
    e2e_mean = float(np.mean(e2e[args.warmup:]))

    # ---------------- dominant-kernel roofline.  Uninstrumented device time of
    # every op's kernels exactly as the TIMED schedule configures them (stage
    # context -> conv tile plan), each op alone with the L2 flushed before it
    # (hios_time_ops: graph = flush -> event -> op kernels -> event, on the
    # launching stream; median of reps).  Cold-L2 and serialised like the ncu
    # launch list of the same kernels (profiles/), so the two agree per launch.
    op_ns = h.hios_time_ops(S, 5, 256 << 20).astype(np.float64)
    if world > 1:
        import torch as _t
        tt = _t.from_numpy(op_ns.copy())
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        op_ns = tt.numpy()
    op_ms = np.where(op_ns > 0, op_ns / 1e6, 0.0)
    F, B = op_work(g, shapes, esz)
    if os.environ.get("HIOS_DUMP"):
        with open(os.environ["HIOS_DUMP"], "w") as f:
            json.dump([{"id": o.id, "name": o.name, "kind": o.kind, "shape": shapes[o.id],
                        "in": [shapes[u] for u in g.preds(o.id)], "k": [o.kh, o.kw, o.sh, o.sw],
                        "ms": float(op_ms[o.id]), "gflop": F[o.id] / 1e9, "mb": B[o.id] / 1e6,
                        "gpu": int(op_gpu[o.id]), "stage": int(op_stage[o.id])} for o in g.ops], f, indent=0)

    # ops of conv_tc_kernel only: 3x3 stride-2 3-channel stems with K <= 40 run
    # on CUDA cores (csrc/exec.cu stem3_conv, conv_stem3_kernel)
    def on_tc(o):
        ci = shapes[g.preds(o.id)[0]][0]
        return not (ci == 3 and o.kh == 3 and o.kw == 3 and o.sh == 2 and o.sw == 2 and o.out_c <= 40)
    conv_ids = [o.id for o in g.ops if o.kind == "conv" and op_ms[o.id] > 0 and on_tc(o)]
    conv_flops = float(F[conv_ids].sum())
    conv_s = float(op_ms[conv_ids].sum()) / 1e3
    all_s = float(op_ms.sum()) / 1e3
    peak_t = pk["bf16_tflops"]
    achieved = conv_flops / conv_s / 1e12 if conv_s > 0 else 0.0
    traffic = None
    tp = os.path.join(ROOT, "profiles", f"conv_traffic_{workload}.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get("bytes_per_launch")
        except Exception:
            traffic = None
    best = max(conv_ids, key=lambda v: F[v] / max(op_ms[v], 1e-9)) if conv_ids else None
    n_launch = max(len(conv_ids), 1)
    roof = {"bound": "tensor", "kernel": "conv_tc_kernel (tcgen05 implicit GEMM)",
            "achieved": achieved, "peak": peak_t, "unit": "TFLOP/s",
            "frac": achieved / peak_t if peak_t else None, "traffic": traffic,
            "traffic_src": (f"profiles/conv_traffic_{workload}.json (ncu dram__bytes_read+write per conv_tc "
                            f"launch, one launch list of this bench command)") if traffic else None,
            "launches_per_step": len(conv_ids),
            "flops_per_launch": conv_flops / n_launch,
            "algorithmic_bytes_per_launch": float(B[conv_ids].sum()) / n_launch,
            "avg_launch_us": conv_s / n_launch * 1e6,
            "share_of_kernel_time": conv_s / all_s if all_s > 0 else None,
            "best_launch": None if best is None else {
                "op": g.ops[best].name, "us": float(op_ms[best] * 1e3),
                "tflops": float(F[best] / (op_ms[best] * 1e-3) / 1e12)},
            "measured_on": ("hios_time_ops: each op of the timed schedule alone (its stage config), "
                            "L2 flushed, CUDA events on the launching stream, median of 5"),
            "peak_src": f"{pk['src']} bf16 burst (kernel timed alone)"}
    mem_ids = [o.id for o in g.ops if o.kind in ("maxpool", "avgpool", "add", "gap") and op_ms[o.id] > 0]
    if mem_ids:
        mb = float(B[mem_ids].sum())
        ms_ = float(op_ms[mem_ids].sum()) / 1e3
        roof["secondary"] = {"bound": "hbm", "kernels": "pool / add / gap kernels (csrc/misc.cu)",
                             "achieved": mb / ms_ / 1e9, "peak": pk["hbm_gbs"], "unit": "GB/s",
                             "frac": mb / ms_ / 1e9 / pk["hbm_gbs"], "launches_per_step": len(mem_ids),
                             "algorithmic_bytes_per_launch": mb / len(mem_ids)}

    cp_s = critical_path_bound(g, F, B, op_gpu, op_stage, M, pk, esz, shapes, args.dtype)
    # single-GPU references measured in the same run (rank 0, N == 1 only)
    extra = {}
    if world == 1:
        # M = 1 also times HIOS-LP / HIOS-MR / LP-inter-only over 2 LOGICAL GPUs
        # aliased on this device (one CUDA graph; a schedule-structure
        # comparison executed on the hardware, not a 2-GPU measurement)
        M2 = M if M > 1 else 2
        for name, (m_, w_) in {"sequential": (1, 1), "ios_style": (1, args.window), "ios": (1, args.window),
                               "lp_inter_only": (M2, 1), "hios_mr": (M2, args.window),
                               "hios_lp_2lgpu": (2, args.window)}.items():
            if name == "hios_lp_2lgpu" and M > 1:
                continue
            t_s0 = time.perf_counter()
            try:
                if name == "hios_mr":
                    Sx = h.hios_schedule_mr(G, m_, w_)
                elif name == "ios":  # exact single-GPU DP, t(S) profiled lazily, bounded
                    Sx = h.hios_schedule_ios(G, w_)
                else:
                    Sx = h.hios_schedule_lp(G, m_, w_)
            except h.HiosError as ex:
                extra[name] = {"unavailable": str(ex)}
                continue
            t_sched_x = time.perf_counter() - t_s0
            h.hios_schedule_stage_mode(Sx, args.stage_mode)
            if m_ > 1:
                ndev = torch.cuda.device_count()
                h.hios_schedule_place(Sx, [i % ndev for i in range(m_)])
            for _ in range(3):
                run_dev(Sx)
            tx = timed_loop(Sx, args.steps)
            extra[name] = {"ms": float(np.mean(tx)),
                           "predicted_ms": h.hios_schedule_latency_ns(Sx) / 1e6,
                           "gpus_used": int(len(set(h.hios_schedule_stages(Sx)[0].tolist()))),
                           "schedule_s": t_sched_x}
            if m_ > 1 and M == 1:
                extra[name]["logical_gpus_aliased_on_one_device"] = m_
            del Sx

    sweep = {}
    if world == 1 and args.sweep and not os.environ.get("HIOS_NCU"):
        for item in [v for v in args.sweep.split(",") if v]:
            spec, dt = (item.split(":") if ":" in item else (item, args.dtype))
            model, sz = (spec.split("@") if "@" in spec else (args.model, spec))
            key = f"{model}@{sz}" + ("" if dt == args.dtype else f":{dt}")
            try:
                sweep[key] = measure_workload(h, torch, model, int(sz), M, args, dev, stream, flush, pk, dt)
            except Exception as ex:  # noqa: BLE001 -- reported, never silently dropped
                sweep[key] = {"error": f"{type(ex).__name__}: {ex}"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        vals, desc, threads = oracle_leg(g, W, x, 2, args.cpu_budget)
        cpu = {"value": float(np.mean(vals)), "unit": "ms", "cores": threads, "kind": "oracle", "sample": desc}

    if rank == 0:
        used = sorted(set(int(a) for a in op_gpu.tolist()))
        line = {
            "metric": METRIC, "value": ms, "unit": "ms", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False, "scaling": "weak",
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic", "config": cfg,
            "roofline": roof,
            "critical_path": {"bound_ms": cp_s * 1e3, "frac": (cp_s * 1e3) / ms if ms > 0 else None,
                              "form": "overlap-edge lower bound, bf16 burst + HBM measured peaks"},
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_ms, "stat": "median", "mean": e2e_mean, "unit": "ms", "h2d_bytes_per_step": int(x.nbytes),
                    "d2h_bytes_per_step": int(n_out * 4), "api": "hios_run (pinned host buffers)"},
            "gpu_launches": int(h.hios_kernel_count(S)) * args.steps,
            "clocks": clocks,
            "schedule": {"kind": f"HIOS-LP M={M} w={args.window}", "gpus_used": len(used),
                         "stages_per_gpu": [int(a) for a in n_stages], "predicted_ms": predicted_ms,
                         "profile_s": t_prof, "schedule_s": t_sched},
            "single_gpu_refs": extra,
            "size_sweep": sweep,
            "wall_s_timed_region": wall,
            "paper": PAPER_NUMBERS,
        }
        if "sequential" in extra:
            line["speedup_vs_sequential"] = extra["sequential"]["ms"] / ms
        if "ios_style" in extra:
            line["speedup_vs_ios_style"] = extra["ios_style"]["ms"] / ms
        if "ms" in extra.get("ios", {}):
            line["speedup_vs_ios"] = extra["ios"]["ms"] / ms
        print(json.dumps(line))
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
