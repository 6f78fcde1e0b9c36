"""Seeded synthetic inputs and random-init weights (SURVEY.md §8(d) recipe).

This module holds NO arithmetic of the method: it only draws random numbers
with fixed seeds.  Both the CPU oracle and the CUDA path receive exactly these
float32 arrays.

  input  x ~ U[0, 1), shape (1, C, H, W), seed 0
  conv   W ~ N(0, 2 / fan_in) (He-normal), shape (K, C, kh, kw), seed 1000 + op id
         (a single-tap conv, op.tap = (r, s): fan_in = C and every other tap zero)
         folded BN: scale ~ U[0.5, 1.5], shift ~ N(0, 0.1^2)  (same generator)
  sepconv  per repetition r: depthwise Wd ~ N(0, 2/(kh*kw)) shape (C, kh, kw),
           pointwise Wp ~ N(0, 2/C) shape (K, C), scale, shift
  linear W ~ N(0, 1/fan_in) shape (K, C); bias ~ N(0, 0.1^2)
  add (agg=1): weights 1/n (a mean of n inputs)
  sepconv (agg=1): positive weights U[0.5, 1.5]/n (RandWire's learned
           weighted input aggregation, Xie et al.; not in PAPER.md)
"""
from __future__ import annotations

from typing import Dict

import numpy as np

from .graphs import GraphSpec


def make_input(g: GraphSpec, seed: int = 0) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.random((1, g.in_c, g.in_h, g.in_w), dtype=np.float64).astype(np.float32)


def make_weights(g: GraphSpec, base_seed: int = 1000) -> Dict[int, Dict[str, np.ndarray]]:
    out: Dict[int, Dict[str, np.ndarray]] = {}
    for op in g.ops:
        rng = np.random.default_rng(base_seed + op.id)
        w: Dict[str, np.ndarray] = {}
        if op.kind == "conv":
            tap = getattr(op, "tap", None)
            fan_in = op.in_c * (1 if tap else op.kh * op.kw)
            w["weight"] = rng.normal(0.0, np.sqrt(2.0 / fan_in),
                                     (op.out_c, op.in_c, op.kh, op.kw)).astype(np.float32)
            if tap:  # single-tap conv: the other taps are structurally zero
                mask = np.zeros((op.kh, op.kw), dtype=np.float32)
                mask[tap[0], tap[1]] = 1.0
                w["weight"] *= mask
            w["scale"] = rng.uniform(0.5, 1.5, op.out_c).astype(np.float32)
            w["shift"] = rng.normal(0.0, 0.1, op.out_c).astype(np.float32)
        elif op.kind == "sepconv":
            c = op.in_c
            dws, pws, scs, shs = [], [], [], []
            for r in range(op.reps):
                dws.append(rng.normal(0.0, np.sqrt(2.0 / (op.kh * op.kw)),
                                      (c, op.kh, op.kw)).astype(np.float32))
                pws.append(rng.normal(0.0, np.sqrt(2.0 / c), (op.out_c, c)).astype(np.float32))
                scs.append(rng.uniform(0.5, 1.5, op.out_c).astype(np.float32))
                shs.append(rng.normal(0.0, 0.1, op.out_c).astype(np.float32))
                c = op.out_c
            w["dw"] = dws
            w["pw"] = pws
            w["scale"] = scs
            w["shift"] = shs
            if op.agg:
                w["agg"] = (rng.uniform(0.5, 1.5, op.n_in) / op.n_in).astype(np.float32)
        elif op.kind == "linear":
            w["weight"] = rng.normal(0.0, np.sqrt(1.0 / op.in_c),
                                     (op.out_c, op.in_c)).astype(np.float32)
            w["shift"] = rng.normal(0.0, 0.1, op.out_c).astype(np.float32)
        elif op.kind == "add" and op.agg:
            w["agg"] = np.full(op.n_in, 1.0 / op.n_in, dtype=np.float32)
        out[op.id] = w
    return out
