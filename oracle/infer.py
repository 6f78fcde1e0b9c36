"""ORACLE -- test infrastructure only.  Plain, slow CPU reference of sequential
DAG-CNN inference.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this module; the product path
(paper_conf_cluster_kundus23_b200) never does.

What it computes.  HIOS only re-orders operators and distributes them over
GPUs (§III), so a scheduled run reaches exactly the result
of plain *sequential* inference ("Sequential scheduling executes the
operator one by one according to a certain topological order in a single
GPU").  The oracle is therefore the plain definition of every operator,
evaluated in topological order, in float64 by default (the paper does not fix
the precision).

Operator definitions (NCHW, batch 1, zero padding):
  conv    y[k,p,q] = act(scale[k] * sum_{c,r,s} x'[c, p*sh-ph+r*dh, q*sw-pw+s*dw]
                                               * W[k,c,r,s] + shift[k])
          x' = relu(x) when the op has pre_relu (NASNet's ReLU -> conv -> BN), else x
          (conv + folded BN + ReLU = one operator)
  sepconv per repetition: a = sum_i agg_i x_i ; a = relu(a) if pre_relu ;
          d[c,p,q] = sum_{r,s} a[c, p*sh-ph+r, q*sw-pw+s] * Wd[c,r,s] ;
          y[k] = scale[k] * sum_c Wp[k,c] d[c] + shift[k] ; relu on the last
          repetition if relu.  (stride on the first repetition only)
  maxpool y[c,p,q] = max over the window of the in-bounds inputs
  avgpool y[c,p,q] = sum over the in-bounds window / divisor; divisor = number
          of window positions inside the padded extent [-ph, H+ph) when
          count_include_pad, else the number of in-bounds positions
  gap     y[c] = mean_{h,w} x[c,h,w]
  linear  y[k] = sum_c W[k,c] x[c] + b[k]
  concat  channel concatenation in input-slot order
  add     y = act(sum_i agg_i x_i)   (agg_i = 1 unless the op carries weights)
  identity y = x
Output size (pools and convs):
  P = floor((H + 2ph - dh(kh-1) - 1)/sh) + 1  (ceil_mode: ceil, and the last
  window must start inside the input or the left padding).
"""
from __future__ import annotations

from typing import Dict, List, Optional

import numpy as np


def out_size(h: int, k: int, s: int, p: int, d: int = 1, ceil_mode: int = 0) -> int:
    num = h + 2 * p - d * (k - 1) - 1
    if ceil_mode:
        o = -(-num // s) + 1
        if (o - 1) * s >= h + p:
            o -= 1
    else:
        o = num // s + 1
    return o


def conv2d(x, W, sh=1, sw=1, ph=0, pw=0, dh=1, dw=1):
    """Direct convolution (cross-correlation) by its definition: the sum over
    (r, s) is written out; the sum over c is one library matrix product."""
    C, H, Wd = x.shape
    K, C2, R, S = W.shape
    assert C == C2
    P = out_size(H, R, sh, ph, dh)
    Q = out_size(Wd, S, sw, pw, dw)
    xp = np.zeros((C, H + 2 * ph, Wd + 2 * pw), dtype=x.dtype)
    xp[:, ph:ph + H, pw:pw + Wd] = x
    y = np.zeros((K, P, Q), dtype=x.dtype)
    for r in range(R):
        for s in range(S):
            patch = xp[:, r * dh: r * dh + sh * (P - 1) + 1: sh,
                       s * dw: s * dw + sw * (Q - 1) + 1: sw]
            y += np.tensordot(W[:, :, r, s], patch, axes=([1], [0]))
    return y


def depthwise2d(x, Wd, sh=1, sw=1, ph=0, pw=0):
    C, H, Wi = x.shape
    _, R, S = Wd.shape
    P = out_size(H, R, sh, ph)
    Q = out_size(Wi, S, sw, pw)
    xp = np.zeros((C, H + 2 * ph, Wi + 2 * pw), dtype=x.dtype)
    xp[:, ph:ph + H, pw:pw + Wi] = x
    y = np.zeros((C, P, Q), dtype=x.dtype)
    for r in range(R):
        for s in range(S):
            y += Wd[:, r, s][:, None, None] * xp[:, r: r + sh * (P - 1) + 1: sh,
                                                  s: s + sw * (Q - 1) + 1: sw]
    return y


def pool2d(x, kind, kh, kw, sh, sw, ph, pw, ceil_mode=0, count_include_pad=1):
    C, H, W = x.shape
    P = out_size(H, kh, sh, ph, 1, ceil_mode)
    Q = out_size(W, kw, sw, pw, 1, ceil_mode)
    y = np.empty((C, P, Q), dtype=x.dtype)
    for p in range(P):
        h0 = p * sh - ph
        for q in range(Q):
            w0 = q * sw - pw
            hs, he = max(h0, 0), min(h0 + kh, H)
            ws, we = max(w0, 0), min(w0 + kw, W)
            win = x[:, hs:he, ws:we]
            if kind == "maxpool":
                y[:, p, q] = win.max(axis=(1, 2))
            else:
                if count_include_pad:
                    div = (min(h0 + kh, H + ph) - h0) * (min(w0 + kw, W + pw) - w0)
                else:
                    div = (he - hs) * (we - ws)
                y[:, p, q] = win.sum(axis=(1, 2)) / div
    return y


def relu(a):
    return np.maximum(a, 0)


def run_op(op, ins: List[np.ndarray], w: Dict, dtype=np.float64) -> np.ndarray:
    k = op.kind
    if k == "conv":
        x = relu(ins[0]) if getattr(op, "pre_relu", 0) else ins[0]
        y = conv2d(x, w["weight"].astype(dtype), op.sh, op.sw, op.ph, op.pw, op.dh, op.dw)
        y = y * w["scale"].astype(dtype)[:, None, None] + w["shift"].astype(dtype)[:, None, None]
        return relu(y) if op.relu else y
    if k == "sepconv":
        if op.agg:
            a = sum(float(wi) * xi for wi, xi in zip(w["agg"].astype(dtype), ins))
        else:
            assert len(ins) == 1
            a = ins[0]
        for r in range(op.reps):
            if op.pre_relu:
                a = relu(a)
            s = (op.sh, op.sw) if r == 0 else (1, 1)
            d = depthwise2d(a, w["dw"][r].astype(dtype), s[0], s[1], op.ph, op.pw)
            y = np.tensordot(w["pw"][r].astype(dtype), d, axes=([1], [0]))
            a = y * w["scale"][r].astype(dtype)[:, None, None] + \
                w["shift"][r].astype(dtype)[:, None, None]
        return relu(a) if op.relu else a
    if k in ("maxpool", "avgpool"):
        return pool2d(ins[0], k, op.kh, op.kw, op.sh, op.sw, op.ph, op.pw,
                      op.ceil_mode, op.count_include_pad)
    if k == "gap":
        return ins[0].mean(axis=(1, 2), keepdims=True)
    if k == "linear":
        v = ins[0].reshape(-1)
        y = w["weight"].astype(dtype) @ v + w["shift"].astype(dtype)
        return y.reshape(-1, 1, 1)
    if k == "concat":
        return np.concatenate(ins, axis=0)
    if k == "add":
        if op.agg:
            y = sum(float(wi) * xi for wi, xi in zip(w["agg"].astype(dtype), ins))
        else:
            y = sum(ins[1:], ins[0].copy())
        return relu(y) if op.relu else y
    if k == "identity":
        return ins[0].copy()
    raise ValueError(f"unknown op kind {k}")


def run_graph(g, weights, x: np.ndarray, dtype=np.float64,
              keep: Optional[set] = None) -> Dict[int, np.ndarray]:
    """Sequential inference in topological order (builders emit ops in a
    topological order; checked here).  Returns {op id: output (C,H,W)}.  With
    ``keep`` only those outputs are retained (memory at high resolution)."""
    inputs: Dict[int, List] = {o.id: [] for o in g.ops}
    for (s, d, slot) in g.edges:
        assert s < d, "oracle evaluates in id order; builders emit topological ids"
        inputs[d].append((slot, s))
    consumers_left = {o.id: 0 for o in g.ops}
    for (s, d, _) in g.edges:
        consumers_left[s] += 1
    vals: Dict[int, np.ndarray] = {}
    out: Dict[int, np.ndarray] = {}
    for op in g.ops:
        if op.kind == "input":
            y = x[0].astype(dtype)
        else:
            ins = [vals[s] for (_, s) in sorted(inputs[op.id])]
            y = run_op(op, ins, weights[op.id], dtype)
        vals[op.id] = y
        if keep is None or op.id in keep:
            out[op.id] = y
        for (_, s) in inputs[op.id]:
            consumers_left[s] -= 1
            if consumers_left[s] == 0 and (keep is not None and s not in keep):
                vals.pop(s, None)
    return out
