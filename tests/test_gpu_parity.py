"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle on the
same seeded inputs.  Tolerances (north star): normwise max relative error
max|y - y_ref| / max|y_ref| <= 2e-2 for bf16, <= 1e-4 for fp32.

Per-op checks feed each op the GPU's own inputs (read back through
hios_read_op_output) so they isolate one kernel's error; end-to-end checks
compare the network output with the oracle's sequential inference."""
import numpy as np
import pytest

from oracle import infer
from workloads import gen, graphs

pytestmark = pytest.mark.gpu

TOL = {"bf16": 2e-2, "f32": 1e-4}


def hios():
    from paper_conf_cluster_kundus23_b200 import hios as h
    return h


def nerr(y, ref):
    den = float(np.abs(ref).max())
    return float(np.abs(np.asarray(y, np.float64) - ref).max()) / (den if den > 0 else 1.0)


def run_graph_gpu(g, W, x, dtype, M=1, w=1, profile=True, costs=None):
    h = hios()
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, dtype, W)
    if profile:
        h.hios_profile(G, [0], 3)
    else:
        for op in g.ops:
            h.hios_set_op_cost(G, op.id, 1000)
        for e in range(g.n_edges):
            h.hios_set_edge_cost(G, e, 1000)
        h.hios_set_group_model(G, 7, 10)
    S = h.hios_schedule_lp(G, M, w)
    y = h.hios_run(S, x)
    return G, S, y


def per_op_check(g, W, S, dtype, skip_kinds=()):
    """Each op's GPU output vs the oracle op evaluated on the GPU's inputs."""
    h = hios()
    outs = {}
    shapes = {}
    G = S.graph
    for op in g.ops:
        shapes[op.id] = h.hios_graph_shape(G, op.id)
        outs[op.id] = h.hios_read_op_output(S, op.id, shapes[op.id]).astype(np.float64)
    worst = {}
    for op in g.ops:
        if op.kind == "input" or op.kind in skip_kinds:
            continue
        ins = [outs[s] for s in g.preds(op.id)]
        ref = infer.run_op(op, ins, W[op.id])
        if h.hios_op_output_relu(S, op.id):  # the consumers' ReLU applied by the producer
            ref = np.maximum(ref, 0.0)
        e = nerr(outs[op.id], ref)
        worst[op.name] = e
        assert e <= TOL[dtype], (op.name, op.kind, e)
    return worst


CONV_CASES = [
    # (C, K, H, W, kh, kw, s, ph, pw)
    (64, 64, 56, 56, 3, 3, 1, 1, 1),
    (3, 32, 75, 75, 3, 3, 2, 0, 0),       # stem: C=3, stride 2, odd size
    (96, 80, 17, 17, 1, 7, 1, 0, 3),      # 1x7
    (80, 192, 17, 19, 7, 1, 1, 3, 0),     # 7x1, K not a power of 2
    (288, 384, 35, 35, 3, 3, 2, 0, 0),    # C tail (288 = 4.5 x 64), stride 2
    (42, 42, 21, 21, 1, 1, 1, 0, 0),      # C, K not multiples of 8
    (192, 320, 9, 9, 3, 3, 2, 0, 0),
    (512, 1000, 13, 13, 1, 1, 1, 0, 0),   # classifier-like, K tail over 256 tiles
    (48, 64, 35, 35, 5, 5, 1, 2, 2),
    # halo mode (stride 1, output width >= 96): shifted-window A descriptors
    (32, 64, 37, 130, 3, 3, 1, 1, 1),
    (48, 64, 21, 125, 5, 5, 1, 2, 2),
    (80, 192, 9, 252, 3, 3, 1, 0, 0),
    (96, 96, 7, 300, 1, 7, 1, 0, 3),
    (64, 80, 13, 100, 7, 1, 1, 3, 0),
    # stride-2 stems with C <= 4 (bf16: space-to-depth + tensor-core conv)
    (3, 96, 61, 229, 7, 7, 2, 0, 0),      # SqueezeNet conv1 shape, odd sizes, halo width
    (3, 96, 45, 260, 3, 3, 2, 1, 1),      # NASNet-like conv0 with padding
    (3, 39, 33, 37, 3, 3, 2, 1, 1),       # RandWire conv1: K = 39 (ragged N), tap mode
    (2, 24, 30, 31, 5, 5, 2, 2, 2),       # C = 2, 5x5 (taps past R, S in W')
    (4, 32, 41, 300, 3, 3, 2, 0, 0),      # C = 4: packed taps (S' = 2 < 4), halo mode
    (3, 64, 300, 35, 5, 5, 2, 2, 2),      # packed taps (S' = 3), tap mode (narrow output)
    # 3x3 stride-2 stems over 3 channels, K <= 40: direct CUDA-core kernel with
    # weights in the parameter bank (odd Q = 2-pixel tail, padding, K < 32, K = 40)
    (3, 32, 64, 301, 3, 3, 2, 1, 1),
    (3, 24, 20, 21, 3, 3, 2, 0, 0),
    (3, 40, 17, 150, 3, 3, 2, 1, 0),
    # virtual-grid halo mode (stride 1, R*S > 1, output width < 96: tiles of 128
    # consecutive positions of the padded-row grid, virtual columns dropped)
    (160, 192, 62, 62, 1, 7, 1, 0, 3),    # Inception Mixed_6 1x7 at 1024^2 (Wh = 68)
    (160, 192, 62, 62, 7, 1, 1, 3, 0),    # 7x1: 10-row box (Wh = 62)
    (448, 384, 30, 30, 3, 3, 1, 1, 1),    # Mixed_7 3x3, K > 128 (staged epilogue), C tail
    (384, 384, 30, 30, 1, 3, 1, 0, 1),
    (384, 384, 30, 30, 3, 1, 1, 1, 0),    # 3x1 (kps 3: its own unrolled tap loop)
    (40, 24, 13, 90, 3, 3, 1, 1, 1),      # Wh = 92, ragged last tile, small K
    (72, 200, 11, 7, 5, 5, 1, 2, 2),      # tiny image: one tile spans the whole output
    (64, 64, 20, 31, 3, 3, 1, 0, 0),      # no padding: Wh = Q + 2
    # row-group halo tiles (two output rows per box; >= 2 x 148 tiles)
    (32, 64, 300, 150, 3, 3, 1, 1, 1),    # resident weights, two accumulator sets
    (64, 192, 300, 200, 3, 3, 1, 1, 1),   # n_tile 192: one accumulator set (nacc 1)
    (48, 64, 201, 300, 5, 5, 1, 2, 2),    # 5x5, odd P (last group half empty)
    (64, 160, 401, 130, 7, 1, 1, 3, 0),   # 7x1 weight ring
    # pixel pairs (1x1, rows >= 192 px: two 128-pixel accumulators per 256-pixel box)
    (192, 64, 150, 509, 1, 1, 1, 0, 0),   # ragged last pair, resident weights
    (288, 96, 160, 600, 1, 1, 1, 0, 0),   # C tail (288 = 4.5 chunks), weight ring
    # C <= 32 (the box reads past C into zero weights) in halo / tap / vgrid modes
    (16, 48, 40, 300, 3, 3, 1, 1, 1),
    (24, 40, 33, 35, 3, 3, 2, 1, 1),
    (32, 96, 30, 30, 3, 3, 1, 1, 1),
    (32, 64, 50, 50, 1, 1, 1, 0, 0),
    # halo mode with resident weights (one N tile, > 148 output tiles per CTA wave)
    (32, 32, 160, 200, 3, 3, 1, 1, 1),
    (64, 80, 150, 130, 1, 1, 1, 0, 0),
]

def test_op_plan_reports_the_conv_tile_plan():
    """hios_op_plan: a tcgen05 conv reports its A-operand mode and N tile; other
    ops report zeros."""
    C, K, H, Wd = 64, 96, 40, 300
    g = graphs.GraphSpec("conv", C, H, Wd)
    x0 = g.input()
    c = g.conv(x0, K, (3, 3), s=1, p=(1, 1), relu=1)
    g.maxpool(c, 3, 2)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    _, S, _ = run_graph_gpu(g, W, x, "bf16", profile=False)
    h = hios()
    p = h.hios_op_plan(S, 1, solo=True)
    assert p["mode"] == 2 and p["n_tile"] % 16 == 0 and p["tiles"] >= 40 and p["stages"] >= 2, p
    assert h.hios_op_plan(S, 2)["mode"] == 0


SEP_CASES = [
    # (C, K, H, W, k, s, n_in, reps)
    (42, 42, 47, 70, 7, 2, 1, 2),         # NASNet stem shape: 7x7 stride 2, C % 16 != 0
    (78, 78, 40, 45, 3, 1, 5, 1),         # RandWire node: 5-input weighted aggregation
    (168, 168, 20, 33, 5, 1, 1, 2),       # NASNet cell: 5x5, several 16-channel slabs
    (20, 24, 19, 37, 4, 2, 2, 1),         # generic kernel size (even), stride 2, aggregation
    (336, 336, 17, 9, 7, 2, 1, 2),        # deep, narrow (tile mostly padding)
    (84, 84, 37, 41, 5, 2, 1, 2),         # register-blocked dw 5x5/s2 (2 rows per thread)
    (30, 32, 50, 19, 3, 2, 3, 1),         # 3x3/s2 with aggregation, C % 8 != 0
    (48, 48, 35, 66, 7, 1, 1, 1),         # 7x7/s1: 16-row CTA tiles, ragged last tile
]


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
@pytest.mark.parametrize("case", SEP_CASES)
def test_sepconv_parity(dtype, case):
    """Depthwise (bf16: register-blocked FHFMA kernel for square 3/5/7 and
    stride 1/2, else smem-tiled; fp32: smem-tiled) + pointwise per
    repetition, per-op check and end to end."""
    C, K, H, Wd, k, s, n_in, reps = case
    g = graphs.GraphSpec("sep", C, H, Wd)
    x0 = g.input()
    ins = [g.conv(x0, C, 1, relu=0) for _ in range(n_in)] if n_in > 1 else [x0]
    g.sepconv(ins, K, k, s=s, pre_relu=1, relu=1, reps=reps)
    W = gen.make_weights(g)
    x = gen.make_input(g) - 0.5
    _, S, y = run_graph_gpu(g, W, x, dtype, profile=False)
    per_op_check(g, W, S, dtype)
    ref = infer.run_graph(g, W, x)[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL[dtype]


POOL_CASES = [
    # (kind, C, H, W, k, s, p, ceil_mode, count_include_pad)
    ("max", 96, 61, 75, 3, 2, 0, 1, 0),     # SqueezeNet: ceil mode, several column tiles
    ("avg", 288, 35, 41, 3, 1, 1, 0, 1),    # Inception avgpool branch
    ("avg", 42, 33, 29, 3, 2, 1, 0, 0),     # NASNet: C % 16 != 0, in-bounds divisor
    ("max", 40, 20, 70, 3, 2, 1, 0, 0),     # padded max
    ("avg", 24, 17, 40, 2, 2, 0, 1, 1),     # generic k (even), ceil + count_include_pad
    ("avg", 42, 31, 37, 3, 1, 1, 0, 0),     # row-streaming s1: channel tail, in-bounds divisor
    ("avg", 128, 400, 400, 3, 1, 1, 0, 1),  # large s1 average: 64-channel CTAs
    ("avg", 168, 200, 203, 3, 1, 1, 0, 0),  # large s1 average, partial last 64-channel group, in-bounds divisor
    ("max", 64, 801, 803, 3, 2, 0, 1, 0),   # row-streaming s2, ceil mode, several rows per strip
    ("max", 20, 9, 9, 3, 1, 1, 0, 0),       # row-streaming s1 max, tiny
]


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
@pytest.mark.parametrize("case", POOL_CASES)
def test_pool_parity(dtype, case):
    kind, C, H, Wd, k, s, p, cm, cip = case
    g = graphs.GraphSpec("pool", C, H, Wd)
    x0 = g.input()
    if kind == "max":
        g.maxpool(x0, k, s, p, ceil_mode=cm)
    else:
        g.avgpool(x0, k, s, p, ceil_mode=cm, count_include_pad=cip)
    W = gen.make_weights(g)
    x = gen.make_input(g) - 0.5
    _, S, y = run_graph_gpu(g, W, x, dtype, profile=False)
    ref = infer.run_graph(g, W, x)[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL[dtype] / (4 if dtype == "bf16" else 1)


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_small_op_zoo(dtype):
    """pools (ceil / pad / count_include_pad), add (weighted, ReLU), concat
    (in-place and copied slices), sepconv (aggregation, reps=2, stride 2),
    gap, linear, identity."""
    g = graphs.GraphSpec("zoo", 24, 23, 23)
    x0 = g.input()
    a = g.conv(x0, 40, 3, p=1)
    b = g.maxpool(a, 3, 2, 1, ceil_mode=1)
    c = g.avgpool(a, 3, 2, 1, count_include_pad=0)
    d = g.avgpool(a, 3, 2, 1, count_include_pad=1)
    e = g.add([b, c, d], relu=1, agg=1)
    f = g.sepconv([b, c], 42, 5, s=1, pre_relu=1, relu=1, reps=2)
    f2 = g.sepconv([e], 40, 3, s=2, pre_relu=1)
    f3 = g.conv(f2, 40, 1, relu=0)
    up = g.maxpool(e, 1, 1)
    cc = g.concat([f, up, e])          # 42-channel slice first: later slices misaligned -> copies
    cc2 = g.concat([g.identity(cc), f])
    gp = g.concat([g.gap(cc2), g.gap(f3)])
    g.linear(gp, 10)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    _, S, y = run_graph_gpu(g, W, x, dtype, profile=False)
    per_op_check(g, W, S, dtype)
    ref = infer.run_graph(g, W, x)[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL[dtype]


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("M,w", [(1, 1), (2, 2), (4, 3)])
def test_tiny_end_to_end(dtype, M, w):
    """configs[0]: Fig.-4-topology conv DAG, 1x64x56x56; multi-GPU schedules run
    on logical GPUs aliased onto cuda:0 (same flags / peer-store code path)."""
    g = graphs.tiny()
    W = gen.make_weights(g)
    x = gen.make_input(g)
    _, S, y = run_graph_gpu(g, W, x, dtype, M=M, w=w)
    ref = infer.run_graph(g, W, x)[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL[dtype]
    per_op_check(g, W, S, dtype)


@pytest.mark.parametrize("name,size", [("inception_v3", 299), ("squeezenet", 224),
                                       ("randwire_ws", 224), ("nasnet_a_large", 331)])
def test_benchmark_end_to_end_bf16(name, size):
    g = graphs.build(name, size)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    _, S, y = run_graph_gpu(g, W, x, "bf16", M=1, w=3)
    per_op_check(g, W, S, "bf16")
    ref = infer.run_graph(g, W, x, keep={g.n_ops - 1})[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL["bf16"]


@pytest.mark.parametrize("name,size", [("inception_v3", 299), ("randwire_ws", 224)])
def test_multi_gpu_schedules_bit_identical(name, size):
    """Placement never changes arithmetic: M = 2, 4, 8 logical GPUs (aliased)
    give bit-identical outputs to the single-GPU sequential schedule."""
    g = graphs.build(name, size)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    _, _, y1 = run_graph_gpu(g, W, x, "bf16", M=1, w=1)
    for M, w in [(2, 2), (4, 3), (8, 3)]:
        _, S, yM = run_graph_gpu(g, W, x, "bf16", M=M, w=w)
        assert np.array_equal(y1, yM), (M, w)


def test_inception_fp32_end_to_end():
    g = graphs.inception_v3(299)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    _, S, y = run_graph_gpu(g, W, x, "f32", M=2, w=2)
    ref = infer.run_graph(g, W, x, keep={g.n_ops - 1})[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL["f32"]


def test_inception_1024_bench_config():
    """configs[1] at full size (1x3x1024x1024) in the bench's launch
    configuration (profiled HIOS-LP, M=1, w=5): logits vs the oracle."""
    g = graphs.inception_v3(1024)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    _, S, y = run_graph_gpu(g, W, x, "bf16", M=1, w=5)
    ref = infer.run_graph(g, W, x, keep={g.n_ops - 1})[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL["bf16"]
    # repeated runs are deterministic
    assert np.array_equal(y, hios().hios_run(S, x))


@pytest.mark.gpu
@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_stem3_concat_slice(dtype):
    """A 3x3 stride-2 3-channel stem with K % 8 != 0 (RandWire conv1-like, K = 39)
    written in place into slot 0 of a concat: its pad channel belongs to the
    next producer, so the kernel must store exactly K channels (csrc/exec.cu:
    kst); next to it the same stem feeding a 1x1 conv from its own buffer."""
    g = graphs.GraphSpec("stem3cat", 3, 45, 70)
    x0 = g.input()
    a = g.conv(x0, 39, 3, s=2, p=1, relu=1)
    b = g.conv(x0, 9, 3, s=2, p=1, relu=1)
    d = g.conv(a, 16, 1, relu=1)
    e = g.conv(x0, 39, 3, s=2, p=1, relu=0)
    f = g.conv(e, 16, 1, relu=1)
    g.concat([a, b, d, f])
    W = gen.make_weights(g)
    x = gen.make_input(g) - 0.5
    _, S, y = run_graph_gpu(g, W, x, dtype, profile=False)
    ref = infer.run_graph(g, W, x)[g.n_ops - 1]
    assert nerr(y.reshape(ref.shape), ref) <= TOL[dtype] / (4 if dtype == "bf16" else 1)


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
@pytest.mark.parametrize("M", [1, 2])
def test_pre_relu_conv_and_factorized_reduction(dtype, M):
    """NASNet pieces: pre-ReLU 1x1 convs sharing one ReLU'd copy of their input
    (made after the producer), the factorized reduction (stride-2 1x1 conv +
    single-tap 3x3/s2/p1 conv + concat) on an odd-sized input, and on M = 2
    logical GPUs the consumer-side ReLU copy of a remote input."""
    g = graphs.GraphSpec("nasfr", 24, 45, 37)
    x0 = g.input()
    a = g.conv(x0, 40, 3, p=1, relu=0)
    f1 = g.conv(a, 32, 1, relu=0, pre_relu=1)
    f2 = g.conv(a, 16, 1, relu=0, pre_relu=1)
    fr = graphs._nas_factorized(g, a, 48, "fr")
    g.concat([g.maxpool(f1, 3, 2, 1), g.maxpool(f2, 3, 2, 1), fr])
    W = gen.make_weights(g)
    x = gen.make_input(g) - 0.5
    h = hios()
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, dtype, W)
    for op in g.ops:
        h.hios_set_op_cost(G, op.id, 0 if op.kind == "input" else 10000)
    for e in range(g.n_edges):
        h.hios_set_edge_cost(G, e, 50)
    h.hios_set_group_model(G, 9, 10)
    S = h.hios_schedule_lp(G, M, 2)
    y = h.hios_run(S, x)
    per_op_check(g, W, S, dtype)
    ref = infer.run_graph(g, W, x)[g.n_ops - 1].reshape(-1)
    assert nerr(y, ref) <= TOL[dtype]
