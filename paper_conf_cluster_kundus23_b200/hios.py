"""Thin ctypes binding of libhios.so (include/hios.h): same function names,
argument marshalling only -- every step of the path runs in the library's
CUDA kernels and host C++.  Importing this module fails loudly if the
extension has not been built (no CPU fallback exists)."""
from __future__ import annotations

import ctypes as C
import os
from typing import Dict, List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# HIOS_LIB: load another build of the library (A/B timing experiments only)
LIB_PATH = os.environ.get("HIOS_LIB", os.path.join(_HERE, "libhios.so"))

KIND = {"input": 0, "conv": 1, "sepconv": 2, "maxpool": 3, "avgpool": 4, "gap": 5,
        "concat": 6, "add": 7, "linear": 8, "identity": 9}
HIOS_F32, HIOS_BF16 = 0, 1
DTYPE = {"f32": HIOS_F32, "fp32": HIOS_F32, "float32": HIOS_F32, "bf16": HIOS_BF16}


class HiosError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"hios status {code}: {msg}")
        self.code = code


class hios_op(C.Structure):
    _fields_ = [("kind", C.c_int32), ("in_c", C.c_int32), ("out_c", C.c_int32),
                ("kh", C.c_int32), ("kw", C.c_int32), ("sh", C.c_int32), ("sw", C.c_int32),
                ("ph", C.c_int32), ("pw", C.c_int32), ("dh", C.c_int32), ("dw", C.c_int32),
                ("relu", C.c_int32), ("pre_relu", C.c_int32), ("ceil_mode", C.c_int32),
                ("count_include_pad", C.c_int32), ("reps", C.c_int32),
                ("weight", C.POINTER(C.c_float)), ("scale", C.POINTER(C.c_float)),
                ("shift", C.POINTER(C.c_float)), ("agg", C.POINTER(C.c_float)),
                ("cost_ns", C.c_int64)]


class hios_edge(C.Structure):
    _fields_ = [("src", C.c_int32), ("dst", C.c_int32), ("slot", C.c_int32),
                ("reserved", C.c_int32), ("cost_ns", C.c_int64)]


_lib = None


def load() -> C.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with "
                          f"`python -c 'import __graft_entry__ as g; g.build()'` (no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    P, I32, I64, VP = C.POINTER, C.c_int32, C.c_int64, C.c_void_p
    sig = {
        "hios_graph_create": [P(hios_op), I32, P(hios_edge), I32, I32, I32, I32, I32, P(VP)],
        "hios_graph_shape": [VP, I32, P(I32), P(I32), P(I32)],
        "hios_set_op_cost": [VP, I32, I64],
        "hios_set_edge_cost": [VP, I32, I64],
        "hios_set_group_cost": [VP, P(I32), I32, I64],
        "hios_set_group_model": [VP, I32, I32],
        "hios_get_costs": [VP, P(I64), P(I64)],
        "hios_group_cost": [VP, P(I32), I32, P(I64)],
        "hios_profile": [VP, P(I32), I32, I32],
        "hios_schedule_lp": [VP, I32, I32, P(VP)],
        "hios_schedule_import": [VP, I32, I32, P(I32), P(I32), P(VP)],
        "hios_schedule_mr": [VP, I32, I32, P(VP)],
        "hios_schedule_ios": [VP, I32, I64, P(VP)],
        "hios_schedule_latency_ns": [VP, P(I64)],
        "hios_schedule_stages": [VP, P(I32), P(I32), P(I32)],
        "hios_schedule_place": [VP, P(I32), I32],
        "hios_schedule_bind_rank": [VP, P(I32), I32, I32],
        "hios_ipc_export": [VP, VP, P(C.c_size_t)],
        "hios_ipc_import": [VP, I32, VP, C.c_size_t],
        "hios_output_numel": [VP, P(I64)],
        "hios_run": [VP, P(C.c_float), P(C.c_float)],
        "hios_run_device": [VP, VP, VP, VP],
        "hios_run_timed": [VP, VP, VP, VP, P(I64)],
        "hios_read_op_output": [VP, I32, P(C.c_float), I64],
        "hios_kernel_count": [VP, P(I64)],
        "hios_op_plan": [VP, I32, I32, P(I32)],
        "hios_op_output_relu": [VP, I32, P(I32)],
        "hios_schedule_stage_mode_used": [VP, P(I32)],
        "hios_time_ops": [VP, I32, I64, P(I64)],
        "hios_schedule_transport": [VP, I32],
        "hios_schedule_stage_mode": [VP, I32],
        "hios_nccl_unique_id": [VP],
        "hios_schedule_nccl_init": [VP, VP, I32, I32],
        "hios_schedule_transfers": [VP, P(I32), P(I32), I32, P(I32)],
    }
    for name, args in sig.items():
        if not hasattr(lib, name):  # an older build (A/B timing via HIOS_LIB)
            continue
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = C.c_int
    lib.hios_graph_destroy.argtypes = [VP]
    lib.hios_graph_destroy.restype = None
    lib.hios_schedule_destroy.argtypes = [VP]
    lib.hios_schedule_destroy.restype = None
    lib.hios_last_error.argtypes = []
    lib.hios_last_error.restype = C.c_char_p
    lib.hios_abi_version.argtypes = []
    lib.hios_abi_version.restype = C.c_int32
    _lib = lib
    return lib


def _ck(st: int):
    if st != 0:
        raise HiosError(st, load().hios_last_error().decode())


def _fptr(a: Optional[np.ndarray]):
    if a is None:
        return None
    return a.ctypes.data_as(C.POINTER(C.c_float))


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


class Graph:
    def __init__(self, handle, n_ops: int, n_edges: int):
        self.h = handle
        self.n_ops = n_ops
        self.n_edges = n_edges

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.hios_graph_destroy(self.h)
            self.h = None


class Schedule:
    def __init__(self, handle, graph: Graph, n_gpus: int):
        self.h = handle
        self.graph = graph  # keeps the Python graph object alive too
        self.n_gpus = n_gpus

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.hios_schedule_destroy(self.h)
            self.h = None


# ------------------------------------------------------------------ graph
def pack_ops(ops: Sequence, weights: Optional[Dict[int, Dict]] = None):
    """Marshal op descriptions (objects with the workload attributes: kind, in_c,
    out_c, kh, ... and optional cost_ns) and their fp32 weights into hios_op."""
    arr = (hios_op * len(ops))()
    keep = []
    for i, o in enumerate(ops):
        a = arr[i]
        a.kind = KIND[o.kind] if isinstance(o.kind, str) else int(o.kind)
        for f in ("in_c", "out_c", "kh", "kw", "sh", "sw", "ph", "pw", "dh", "dw", "relu",
                  "pre_relu", "ceil_mode", "reps"):
            setattr(a, f, int(getattr(o, f, 0) or 0))
        a.count_include_pad = int(getattr(o, "count_include_pad", 1))
        a.cost_ns = int(getattr(o, "cost_ns", -1) if getattr(o, "cost_ns", None) is not None else -1)
        w = (weights or {}).get(getattr(o, "id", i), {})
        wt = sc = sh = ag = None
        if a.kind == KIND["sepconv"] and "dw" in w:
            parts = []
            for r in range(len(w["dw"])):
                parts += [w["dw"][r].ravel(), w["pw"][r].ravel()]
            wt = np.concatenate(parts).astype(np.float32)
            sc = np.concatenate(w["scale"]).astype(np.float32)
            sh = np.concatenate(w["shift"]).astype(np.float32)
        else:
            if "weight" in w:
                wt = np.ascontiguousarray(w["weight"], dtype=np.float32).ravel()
            if "scale" in w:
                sc = np.ascontiguousarray(w["scale"], dtype=np.float32)
            if "shift" in w:
                sh = np.ascontiguousarray(w["shift"], dtype=np.float32)
        if "agg" in w:
            ag = np.ascontiguousarray(w["agg"], dtype=np.float32)
        _check_sizes(a, wt, sc, sh, ag, getattr(o, "n_in", None))
        for x in (wt, sc, sh, ag):
            if x is not None:
                keep.append(x)
        a.weight, a.scale, a.shift, a.agg = _fptr(wt), _fptr(sc), _fptr(sh), _fptr(ag)
    return arr, keep


def _check_sizes(a, wt, sc, sh, ag, n_in):
    """The library copies fixed counts from these arrays (include/hios.h hios_op
    weight layouts): a wrongly sized array would be an out-of-bounds read."""
    k = a.kind
    exp = {}
    if k == KIND["conv"]:
        exp = {"weight": a.out_c * a.in_c * a.kh * a.kw, "scale": a.out_c, "shift": a.out_c}
    elif k == KIND["sepconv"]:
        reps = max(a.reps, 1)
        tot, c = 0, a.in_c
        for _ in range(reps):
            tot += c * a.kh * a.kw + a.out_c * c
            c = a.out_c
        exp = {"weight": tot, "scale": reps * a.out_c, "shift": reps * a.out_c}
    elif k == KIND["linear"]:
        exp = {"weight": a.out_c * a.in_c, "shift": a.out_c}
    for name, arr in (("weight", wt), ("scale", sc), ("shift", sh)):
        if arr is not None and name in exp and arr.size != exp[name]:
            raise HiosError(1, f"op kind {k}: {name} has {arr.size} elements, expected {exp[name]}")
    if ag is not None and n_in is not None and ag.size != int(n_in):
        raise HiosError(1, f"op kind {k}: agg has {ag.size} elements, expected {n_in} (one per input)")


def pack_edges(edges: Sequence, costs: Optional[Sequence[int]] = None):
    arr = (hios_edge * len(edges))()
    for i, e in enumerate(edges):
        src, dst, slot = e[0], e[1], e[2]
        arr[i].src, arr[i].dst, arr[i].slot = int(src), int(dst), int(slot)
        arr[i].cost_ns = int(costs[i]) if costs is not None else -1
    return arr


def hios_graph_create(ops, edges, in_c: int, in_h: int, in_w: int, dtype="bf16",
                      weights=None, edge_costs=None) -> Graph:
    lib = load()
    oa, keep = pack_ops(ops, weights)
    ea = pack_edges(edges, edge_costs)
    h = C.c_void_p()
    _ck(lib.hios_graph_create(oa, len(ops), ea, len(edges), in_c, in_h, in_w,
                              DTYPE[dtype] if isinstance(dtype, str) else int(dtype), C.byref(h)))
    del keep
    gr = Graph(h, len(ops), len(edges))
    gr.in_numel = int(in_c) * int(in_h) * int(in_w)
    return gr


def hios_graph_shape(g: Graph, op: int):
    c, h, w = C.c_int32(), C.c_int32(), C.c_int32()
    _ck(load().hios_graph_shape(g.h, op, C.byref(c), C.byref(h), C.byref(w)))
    return c.value, h.value, w.value


def hios_set_op_cost(g: Graph, op: int, ns: int):
    _ck(load().hios_set_op_cost(g.h, op, int(ns)))


def hios_set_edge_cost(g: Graph, e: int, ns: int):
    _ck(load().hios_set_edge_cost(g.h, e, int(ns)))


def hios_set_group_cost(g: Graph, ops: Sequence[int], ns: int):
    a = _i32(ops)
    _ck(load().hios_set_group_cost(g.h, a.ctypes.data_as(C.POINTER(C.c_int32)), len(a), int(ns)))


def hios_set_group_model(g: Graph, num: int, den: int):
    _ck(load().hios_set_group_model(g.h, num, den))


def hios_get_costs(g: Graph):
    o = np.zeros(g.n_ops, dtype=np.int64)
    e = np.zeros(max(g.n_edges, 1), dtype=np.int64)
    _ck(load().hios_get_costs(g.h, o.ctypes.data_as(C.POINTER(C.c_int64)),
                              e.ctypes.data_as(C.POINTER(C.c_int64))))
    return o, e[:g.n_edges]


def hios_group_cost(g: Graph, ops: Sequence[int]) -> int:
    a = _i32(ops)
    ns = C.c_int64(0)
    _ck(load().hios_group_cost(g.h, a.ctypes.data_as(C.POINTER(C.c_int32)), len(a), C.byref(ns)))
    return ns.value


def hios_profile(g: Graph, devices: Sequence[int] = (0,), reps: int = 10):
    d = _i32(devices)
    _ck(load().hios_profile(g.h, d.ctypes.data_as(C.POINTER(C.c_int32)), len(d), reps))


# --------------------------------------------------------------- schedule
def hios_schedule_lp(g: Graph, n_gpus: int, window: int) -> Schedule:
    h = C.c_void_p()
    _ck(load().hios_schedule_lp(g.h, n_gpus, window, C.byref(h)))
    return Schedule(h, g, n_gpus)


def hios_schedule_mr(g: Graph, n_gpus: int, window: int) -> Schedule:
    h = C.c_void_p()
    _ck(load().hios_schedule_mr(g.h, n_gpus, window, C.byref(h)))
    return Schedule(h, g, n_gpus)


def hios_schedule_ios(g: Graph, window: int, max_states: int = 0) -> Schedule:
    h = C.c_void_p()
    _ck(load().hios_schedule_ios(g.h, window, int(max_states), C.byref(h)))
    return Schedule(h, g, 1)


def hios_schedule_import(g: Graph, n_gpus: int, window: int, op_gpu, op_stage) -> Schedule:
    a, b = _i32(op_gpu), _i32(op_stage)
    h = C.c_void_p()
    _ck(load().hios_schedule_import(g.h, n_gpus, window, a.ctypes.data_as(C.POINTER(C.c_int32)),
                                    b.ctypes.data_as(C.POINTER(C.c_int32)), C.byref(h)))
    return Schedule(h, g, n_gpus)


def hios_schedule_latency_ns(s: Schedule) -> int:
    v = C.c_int64()
    _ck(load().hios_schedule_latency_ns(s.h, C.byref(v)))
    return v.value


def hios_schedule_stages(s: Schedule):
    n = s.graph.n_ops
    g = np.zeros(n, dtype=np.int32)
    st = np.zeros(n, dtype=np.int32)
    ns = np.zeros(s.n_gpus, dtype=np.int32)
    P = C.POINTER(C.c_int32)
    _ck(load().hios_schedule_stages(s.h, g.ctypes.data_as(P), st.ctypes.data_as(P), ns.ctypes.data_as(P)))
    return g, st, ns


def stages_to_Q(s: Schedule) -> List[List[tuple]]:
    """Q = per-GPU list of stages (tuples of sorted op ids), P:90 notation."""
    g, st, ns = hios_schedule_stages(s)
    Q = [[[] for _ in range(int(ns[i]))] for i in range(s.n_gpus)]
    for v in range(len(g)):
        Q[g[v]][st[v]].append(v)
    return [[tuple(sorted(S)) for S in q] for q in Q]


def hios_schedule_place(s: Schedule, devices: Sequence[int]):
    d = _i32(devices)
    _ck(load().hios_schedule_place(s.h, d.ctypes.data_as(C.POINTER(C.c_int32)), len(d)))


def hios_schedule_bind_rank(s: Schedule, owner: Sequence[int], rank: int):
    d = _i32(owner)
    _ck(load().hios_schedule_bind_rank(s.h, d.ctypes.data_as(C.POINTER(C.c_int32)), len(d), rank))


TRANSPORT = {"peer": 0, "copy": 1, "nccl": 2}


def hios_schedule_transport(s: Schedule, transport):
    t = TRANSPORT[transport] if isinstance(transport, str) else int(transport)
    _ck(load().hios_schedule_transport(s.h, t))


STAGE_MODE = {"streams": 0, "grouped": 1, "dataflow": 2, "auto": 3}


def hios_schedule_stage_mode(s: Schedule, mode):
    m = STAGE_MODE[mode] if isinstance(mode, str) else int(mode)
    _ck(load().hios_schedule_stage_mode(s.h, m))


def hios_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _ck(load().hios_nccl_unique_id(buf))
    return buf.raw


def hios_schedule_nccl_init(s: Schedule, uid: bytes, nranks: int, rank: int):
    assert len(uid) == 128
    buf = C.create_string_buffer(uid, 128)
    _ck(load().hios_schedule_nccl_init(s.h, buf, nranks, rank))


def hios_schedule_transfers(s: Schedule):
    """[(producer op, consumer logical GPU)] in the NCCL transport's global order."""
    n = C.c_int32()
    _ck(load().hios_schedule_transfers(s.h, None, None, 0, C.byref(n)))
    a = np.zeros(max(n.value, 1), dtype=np.int32)
    b = np.zeros(max(n.value, 1), dtype=np.int32)
    _ck(load().hios_schedule_transfers(s.h, a.ctypes.data_as(C.POINTER(C.c_int32)),
                                       b.ctypes.data_as(C.POINTER(C.c_int32)), len(a), C.byref(n)))
    return [(int(a[i]), int(b[i])) for i in range(n.value)]


def hios_ipc_export(s: Schedule) -> bytes:
    n = C.c_size_t(0)
    _ck(load().hios_ipc_export(s.h, None, C.byref(n)))
    buf = C.create_string_buffer(n.value)
    _ck(load().hios_ipc_export(s.h, buf, C.byref(n)))
    return buf.raw[:n.value]


def hios_ipc_import(s: Schedule, rank: int, blob: bytes):
    buf = C.create_string_buffer(blob, len(blob))
    _ck(load().hios_ipc_import(s.h, rank, buf, len(blob)))


def hios_output_numel(s: Schedule) -> int:
    v = C.c_int64()
    _ck(load().hios_output_numel(s.h, C.byref(v)))
    return v.value


# -------------------------------------------------------------------- run
def hios_run(s: Schedule, x: Optional[np.ndarray]) -> np.ndarray:
    out = np.zeros(hios_output_numel(s), dtype=np.float32)
    xin = None if x is None else np.ascontiguousarray(x, dtype=np.float32)
    want = getattr(s.graph, "in_numel", None)
    if xin is not None and want is not None and xin.size != want:
        raise HiosError(1, f"input has {xin.size} elements, expected in_c*in_h*in_w = {want}")
    _ck(load().hios_run(s.h, _fptr(xin), _fptr(out)))
    return out


def hios_run_device(s: Schedule, d_in: int, d_out: int, stream: int = 0):
    _ck(load().hios_run_device(s.h, C.c_void_p(d_in), C.c_void_p(d_out), C.c_void_p(stream)))


def hios_run_timed(s: Schedule, d_in: int, d_out: int, stream: int = 0) -> np.ndarray:
    t = np.zeros(s.graph.n_ops, dtype=np.int64)
    _ck(load().hios_run_timed(s.h, C.c_void_p(d_in), C.c_void_p(d_out), C.c_void_p(stream),
                              t.ctypes.data_as(C.POINTER(C.c_int64))))
    return t


def hios_time_ops(s: Schedule, reps: int = 5, flush_bytes: int = 256 << 20) -> np.ndarray:
    t = np.zeros(s.graph.n_ops, dtype=np.int64)
    _ck(load().hios_time_ops(s.h, reps, flush_bytes, t.ctypes.data_as(C.POINTER(C.c_int64))))
    return t


def hios_read_op_output(s: Schedule, op: int, shape) -> np.ndarray:
    n = int(np.prod(shape))
    out = np.zeros(n, dtype=np.float32)
    _ck(load().hios_read_op_output(s.h, op, _fptr(out), n))
    return out.reshape(shape)


def hios_kernel_count(s: Schedule) -> int:
    v = C.c_int64()
    _ck(load().hios_kernel_count(s.h, C.byref(v)))
    return v.value


def hios_schedule_stage_mode_used(s: Schedule) -> str:
    """The stage mode the schedule's graphs execute (AUTO resolved after the first run)."""
    v = C.c_int32()
    _ck(load().hios_schedule_stage_mode_used(s.h, C.byref(v)))
    return {m: k for k, m in STAGE_MODE.items()}[v.value]


def hios_op_output_relu(s: Schedule, op: int) -> bool:
    """True when op's stored output is ReLU'd (its consumers' ReLU hoisted into it)."""
    v = C.c_int32()
    _ck(load().hios_op_output_relu(s.h, op, C.byref(v)))
    return bool(v.value)


def hios_op_plan(s: Schedule, op: int, solo: bool = False) -> dict:
    """The tcgen05 conv tile plan of `op` (hios_op_plan); mode 0 = no tcgen05 conv."""
    v = (C.c_int32 * 8)()
    _ck(load().hios_op_plan(s.h, op, 1 if solo else 0, v))
    keys = ("mode", "n_tile", "tiles", "epilogue", "st256", "rows", "stages", "kps")
    return dict(zip(keys, list(v)))


def hios_abi_version() -> int:
    return load().hios_abi_version()
