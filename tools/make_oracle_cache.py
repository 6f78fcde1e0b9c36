#!/usr/bin/env python
"""Write the cached oracle outputs used by the full-size GPU parity tests
(tests/test_gpu_fullsize.py).  Calls only oracle/ (and the seeded workload
generators): no value here ever comes from the CUDA path.

For one (model, input size, seed) the cache holds
  * the network output (the unique sink: the logits), fp64, in full;
  * for a few intermediate operators spread over the topological order
    (`sample_ops`), the oracle value at 4096 flat NCHW positions drawn with a
    fixed seed, plus max|y| over the WHOLE tensor -- the denominator of the
    normwise-max metric, so the test computes
    max_{i in sample} |y_i - yhat_i| / max_all |yhat|.

Usage:  python tools/make_oracle_cache.py inception_v3@2048 squeezenet@2048 ...
Output: tests/golden/oracle_cache/<model>_<size>_s0.npz
(fp64 numpy on the host cores; Inception-v3 at 4096^2 takes minutes.)
"""
from __future__ import annotations

import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import infer  # noqa: E402
from workloads import gen, graphs  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "oracle_cache")
N_SAMPLE = 4096


def sample_ops(g):
    """Six operators at 1/7 .. 6/7 of the topological order (non-input), and
    the sink.  Deterministic in the graph only."""
    ids = [o.id for o in g.ops if o.kind != "input"]
    pick = sorted({ids[int(len(ids) * k / 7)] for k in range(1, 7)})
    sink = g.sinks()[0]
    return [v for v in pick if v != sink] + [sink]


def main(argv):
    os.makedirs(OUT, exist_ok=True)
    for item in argv:
        model, size = item.split("@")
        size = int(size)
        g = graphs.build(model, size)
        W = gen.make_weights(g)
        x = gen.make_input(g)
        ops = sample_ops(g)
        t0 = time.time()
        vals = infer.run_graph(g, W, x, keep=set(ops))
        el = time.time() - t0
        rec = {"model": np.array(model), "size": np.array(size), "seed": np.array(0),
               "ops": np.array(ops, dtype=np.int64),
               "names": np.array([g.ops[v].name for v in ops]),
               "oracle_s": np.array(el)}
        sink = g.sinks()[0]
        for v in ops:
            y = vals[v].reshape(-1)
            rec[f"absmax_{v}"] = np.array(np.abs(y).max())
            rec[f"shape_{v}"] = np.array(vals[v].shape, dtype=np.int64)
            if v == sink:
                rec[f"idx_{v}"] = np.arange(y.size, dtype=np.int64)
            else:
                rng = np.random.default_rng(10_000 + v)
                rec[f"idx_{v}"] = np.sort(rng.choice(y.size, size=min(N_SAMPLE, y.size), replace=False))
            rec[f"val_{v}"] = y[rec[f"idx_{v}"]].astype(np.float64)
        path = os.path.join(OUT, f"{model}_{size}_s0.npz")
        np.savez_compressed(path, **rec)
        print(f"{item}: {len(ops)} ops cached in {el:.1f} s -> {os.path.relpath(path, ROOT)}", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:])
