"""GPU parity at every input size bench.py times ("from the default size
to the largest size"), in bench.py's launch configuration: the graph profiled
on cuda:0 (hios_profile, 5 reps), then HIOS-LP with M = 1, w = 5 through
hios_run.  The fp64 oracle outputs are cached (tests/golden/oracle_cache/,
written by tools/make_oracle_cache.py, which calls only oracle/): the logits in
full, and for six intermediate operators 4096 sampled NCHW elements with the
whole tensor's max|y|.  Checks (normwise-max metric of SURVEY C22):

* network output (the logits) vs the cached end-to-end oracle: <= 2e-2 (bf16);
* each sampled intermediate operator in isolation: the oracle operator
  (oracle/infer.py run_op) evaluated on the GPU's own inputs of that operator
  (read back through hios_read_op_output) vs the GPU output: <= 2e-2;
* the end-to-end drift of those intermediates vs the cached oracle values
  (bf16 storage of every activation through up to ~370 operators) is reported
  and bounded by 5e-2.
"""
import os

import numpy as np
import pytest

from workloads import gen, graphs

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))
CACHE = os.path.join(HERE, "golden", "oracle_cache")
TOL_BF16 = 2e-2

BENCH_CONFIGS = [("inception_v3", 2048), ("inception_v3", 4096), ("randwire_ws", 2048),
                 ("nasnet_a_large", 2048), ("squeezenet", 2048)]


def _cache(model, size):
    path = os.path.join(CACHE, f"{model}_{size}_s0.npz")
    if not os.path.exists(path):
        pytest.fail(f"missing oracle cache {path}: run tools/make_oracle_cache.py {model}@{size}")
    return np.load(path)


@pytest.mark.parametrize("model,size", BENCH_CONFIGS)
def test_bench_config_vs_cached_oracle(model, size):
    from paper_conf_cluster_kundus23_b200 import hios as h
    c = _cache(model, size)
    g = graphs.build(model, size)
    assert int(c["size"]) == size and [g.ops[v].name for v in c["ops"]] == list(c["names"])
    W = gen.make_weights(g)
    x = gen.make_input(g)
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
    h.hios_profile(G, [0], 5)
    S = h.hios_schedule_lp(G, 1, 5)
    y = h.hios_run(S, x)
    from oracle import infer
    sink = g.sinks()[0]
    drift, iso = {}, {}
    for v in c["ops"]:
        v = int(v)
        shape = tuple(int(a) for a in c[f"shape_{v}"])
        full = np.asarray(y if v == sink else h.hios_read_op_output(S, v, shape), np.float64)
        yv = full.reshape(-1)[c[f"idx_{v}"]]
        # an op storing its consumers' ReLU (hios_op_output_relu) is compared with ReLU(oracle)
        relu_v = v != sink and h.hios_op_output_relu(S, v)
        val = np.maximum(c[f"val_{v}"], 0.0) if relu_v else c[f"val_{v}"]
        drift[g.ops[v].name] = float(np.abs(yv - val).max() / float(c[f"absmax_{v}"]))
        if v != sink:
            ins = []
            for u in g.preds(v):
                ins.append(np.asarray(h.hios_read_op_output(S, u, tuple(h.hios_graph_shape(G, u))), np.float64))
            ref = infer.run_op(g.ops[v], ins, W[v]).reshape(-1)
            if relu_v:
                ref = np.maximum(ref, 0.0)
            iso[g.ops[v].name] = float(np.abs(full.reshape(-1) - ref).max() / float(np.abs(ref).max()))
    print(model, size, "end-to-end drift", {k: f"{e:.2e}" for k, e in drift.items()},
          "isolated", {k: f"{e:.2e}" for k, e in iso.items()})
    assert drift[g.ops[sink].name] <= TOL_BF16, drift
    bad = {k: e for k, e in iso.items() if not e <= TOL_BF16}
    assert not bad, bad
    bad = {k: e for k, e in drift.items() if not e <= 5e-2}
    assert not bad, bad
