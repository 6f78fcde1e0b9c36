"""GPU parity at every input size bench.py times ("from the default size
to the largest size"), in bench.py's launch configuration: the graph profiled
on cuda:0 (hios_profile, 5 reps), then HIOS-LP with M = 1, w = 5 through
hios_run.  The fp64 oracle outputs are cached (tests/golden/oracle_cache/,
written by tools/make_oracle_cache.py, which calls only oracle/): the logits in
full, and for six intermediate operators 4096 sampled NCHW elements with the
whole tensor's max|y|, so each check is the normwise-max metric of SURVEY C22
restricted to the sample: max_i |y_i - yhat_i| / max_all |yhat| <= 2e-2 (bf16).
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
    errs = {}
    for v in c["ops"]:
        v = int(v)
        shape = tuple(int(a) for a in c[f"shape_{v}"])
        yv = y if v == g.sinks()[0] else h.hios_read_op_output(S, v, shape)
        yv = np.asarray(yv, np.float64).reshape(-1)[c[f"idx_{v}"]]
        errs[g.ops[v].name] = float(np.abs(yv - c[f"val_{v}"]).max() / float(c[f"absmax_{v}"]))
    print(model, size, {k: f"{e:.2e}" for k, e in errs.items()})
    bad = {k: e for k, e in errs.items() if not e <= TOL_BF16}
    assert not bad, bad
