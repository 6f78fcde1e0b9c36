"""Pins for the inference oracle (oracle/infer.py) against textbook and
library routines independent of it: scipy.signal.correlate, PyTorch CPU fp64
functional ops, torchvision's Inception-v3 / SqueezeNet 1.0 with the same
weights, hand-computed values."""
import numpy as np
import pytest
import torch
import torch.nn.functional as F
from scipy import signal

from oracle import infer as I
from workloads import gen, graphs

torch.set_num_threads(8)


def test_conv_hand_computed_3x3():
    # x = 1..9 on a 3x3 grid, W = all ones 3x3, pad 1: each output = sum of the
    # in-bounds 3x3 neighbourhood.
    x = np.arange(1, 10, dtype=np.float64).reshape(1, 3, 3)
    W = np.ones((1, 1, 3, 3))
    y = I.conv2d(x, W, 1, 1, 1, 1)
    expect = np.array([[12, 21, 16], [27, 45, 33], [24, 39, 28]], dtype=np.float64)
    assert np.array_equal(y[0], expect)
    # stride 2, no pad on a 5x5 ramp with a delta kernel picks x[2p+1, 2q+1]
    x = np.arange(25, dtype=np.float64).reshape(1, 5, 5)
    W = np.zeros((1, 1, 3, 3)); W[0, 0, 1, 1] = 1
    assert np.array_equal(I.conv2d(x, W, 2, 2, 0, 0)[0], x[0, 1:4:2, 1:4:2])


@pytest.mark.parametrize("case", [
    (3, 4, 11, 13, 3, 3, 1, 1, 1, 1, 1, 1),
    (5, 2, 9, 9, 1, 7, 1, 1, 0, 3, 1, 1),
    (4, 3, 12, 10, 7, 1, 2, 2, 3, 0, 1, 1),
    (2, 3, 15, 14, 5, 5, 2, 3, 2, 1, 1, 1),
    (3, 2, 13, 13, 3, 3, 1, 1, 2, 2, 2, 2),
])
def test_conv_vs_scipy_correlate(case):
    C, K, H, W, R, S, sh, sw, ph, pw, dh, dw = case
    rng = np.random.default_rng(7)
    x = rng.standard_normal((C, H, W))
    Wt = rng.standard_normal((K, C, R, S))
    y = I.conv2d(x, Wt, sh, sw, ph, pw, dh, dw)
    xp = np.pad(x, ((0, 0), (ph, ph), (pw, pw)))
    for k in range(K):
        # dilated kernel, then 'valid' correlation and stride subsampling
        kd = np.zeros((C, dh * (R - 1) + 1, dw * (S - 1) + 1))
        kd[:, ::dh, ::dw] = Wt[k]
        full = signal.correlate(xp, kd, mode="valid")[0]
        ref = full[::sh, ::sw]
        assert ref.shape == y[k].shape
        np.testing.assert_allclose(y[k], ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("kind,k,s,p,ceil,cip", [
    ("maxpool", 3, 2, 0, 0, 1), ("maxpool", 3, 2, 0, 1, 1), ("maxpool", 3, 2, 1, 0, 1),
    ("avgpool", 3, 1, 1, 0, 1), ("avgpool", 3, 1, 1, 0, 0), ("avgpool", 3, 2, 1, 0, 0),
    ("avgpool", 3, 2, 1, 1, 1), ("maxpool", 2, 2, 0, 1, 1),
])
def test_pool_vs_torch(kind, k, s, p, ceil, cip):
    rng = np.random.default_rng(3)
    for (H, W) in [(13, 13), (14, 11), (7, 8)]:
        x = rng.standard_normal((5, H, W))
        y = I.pool2d(x, kind, k, k, s, s, p, p, ceil, cip)
        t = torch.from_numpy(x)[None]
        if kind == "maxpool":
            ref = F.max_pool2d(t, k, s, p, ceil_mode=bool(ceil))
        else:
            ref = F.avg_pool2d(t, k, s, p, ceil_mode=bool(ceil), count_include_pad=bool(cip))
        np.testing.assert_allclose(y, ref[0].numpy(), rtol=1e-12, atol=1e-12)


def test_pool_brute_force_python_loops():
    rng = np.random.default_rng(4)
    x = rng.standard_normal((2, 6, 7))
    y = I.pool2d(x, "avgpool", 3, 3, 2, 2, 1, 1, 0, 0)
    for c in range(2):
        for p in range(y.shape[1]):
            for q in range(y.shape[2]):
                vals = [x[c, h, w] for h in range(2 * p - 1, 2 * p + 2)
                        for w in range(2 * q - 1, 2 * q + 2) if 0 <= h < 6 and 0 <= w < 7]
                assert abs(y[c, p, q] - sum(vals) / len(vals)) < 1e-12


def test_out_size_matches_torch_ceil_rule():
    for H in range(5, 40):
        for k, s, p in [(3, 2, 0), (3, 2, 1), (2, 2, 0), (7, 2, 3)]:
            for ceil in (0, 1):
                t = F.max_pool2d(torch.zeros(1, 1, H, H), k, s, p, ceil_mode=bool(ceil))
                assert I.out_size(H, k, s, p, 1, ceil) == t.shape[-1]


def test_sepconv_vs_torch_grouped_conv():
    g = graphs.GraphSpec("t", 6, 9, 9)
    x0 = g.input()
    a = g.conv(x0, 8, 1, relu=0)
    b = g.conv(x0, 8, 1, relu=0)
    s = g.sepconv([a, b], 12, 5, s=2, pre_relu=1, relu=1, reps=2)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    out = I.run_graph(g, W, x)
    ta = torch.from_numpy(out[a])[None]
    tb = torch.from_numpy(out[b])[None]
    w = W[s]
    h = float(w["agg"][0]) * ta + float(w["agg"][1]) * tb
    for r in range(2):
        h = F.relu(h)
        st = 2 if r == 0 else 1
        h = F.conv2d(h, torch.from_numpy(w["dw"][r].astype(np.float64))[:, None],
                     stride=st, padding=2, groups=h.shape[1])
        h = F.conv2d(h, torch.from_numpy(w["pw"][r].astype(np.float64))[:, :, None, None])
        h = h * torch.from_numpy(w["scale"][r].astype(np.float64))[None, :, None, None] + \
            torch.from_numpy(w["shift"][r].astype(np.float64))[None, :, None, None]
    h = F.relu(h)
    np.testing.assert_allclose(out[s], h[0].numpy(), rtol=1e-10, atol=1e-10)


def _load_torchvision(model, g, W):
    """Copy the seeded weights into a torchvision model: conv.weight = W,
    BN(eval) with mean 0, var 1 - eps -> y = scale * x + shift."""
    name2op = {o.name: o for o in g.ops}
    mods = dict(model.named_modules())
    for name, op in name2op.items():
        if op.kind == "conv":
            m = mods[name]
            w = W[op.id]
            if hasattr(m, "conv"):  # BasicConv2d (conv + bn)
                m.conv.weight.data = torch.from_numpy(w["weight"].astype(np.float64))
                eps = m.bn.eps
                m.bn.weight.data = torch.from_numpy(w["scale"].astype(np.float64))
                m.bn.bias.data = torch.from_numpy(w["shift"].astype(np.float64))
                m.bn.running_mean.data = torch.zeros(op.out_c, dtype=torch.float64)
                m.bn.running_var.data = torch.full((op.out_c,), 1.0 - eps, dtype=torch.float64)
            else:  # plain conv with bias (SqueezeNet): fold the scale into W
                m.weight.data = torch.from_numpy(
                    (w["weight"].astype(np.float64) * w["scale"].astype(np.float64)[:, None, None, None]))
                m.bias.data = torch.from_numpy(w["shift"].astype(np.float64))
        elif op.kind == "linear":
            m = mods[name]
            m.weight.data = torch.from_numpy(W[op.id]["weight"].astype(np.float64))
            m.bias.data = torch.from_numpy(W[op.id]["shift"].astype(np.float64))


def test_inception_v3_vs_torchvision():
    import torchvision
    g = graphs.inception_v3(299)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    out = I.run_graph(g, W, x, keep={g.n_ops - 1})
    m = torchvision.models.inception_v3(weights=None, aux_logits=False, init_weights=False)
    m = m.double().eval()
    _load_torchvision(m, g, W)
    with torch.no_grad():
        ref = m(torch.from_numpy(x.astype(np.float64)))
    y = out[g.n_ops - 1].reshape(-1)
    np.testing.assert_allclose(y, ref[0].numpy(), rtol=1e-9, atol=1e-9 * np.abs(y).max())


def test_squeezenet_vs_torchvision():
    import torchvision
    g = graphs.squeezenet(224)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    out = I.run_graph(g, W, x, keep={g.n_ops - 1})
    m = torchvision.models.squeezenet1_0(weights=None).double().eval()
    _load_torchvision(m, g, W)
    with torch.no_grad():
        ref = m(torch.from_numpy(x.astype(np.float64)))
    y = out[g.n_ops - 1].reshape(-1)
    np.testing.assert_allclose(y, ref[0].numpy(), rtol=1e-9, atol=1e-9 * np.abs(y).max())


def test_graph_counts_vs_paper():
    """Inception-v3 has 119 operators and 153 dependencies (input
    placeholder + 94 conv + 13 pools + 11 concats, C20)."""
    g = graphs.inception_v3(299, head=False)
    assert (g.n_ops, g.n_edges) == (119, 153)
    kinds = [o.kind for o in g.ops]
    assert kinds.count("conv") == 94 and kinds.count("concat") == 11
    assert kinds.count("maxpool") + kinds.count("avgpool") == 13
    # NASNet 374 ops / 576 deps; this IR is within 3 %
    n = graphs.nasnet_a_large(331)
    assert abs(n.n_ops - 374) / 374 < 0.03 and abs(n.n_edges - 576) / 576 < 0.03


def test_all_workloads_run_small():
    for name, size in [("tiny", None), ("randwire_ws", 64), ("nasnet_a_large", 64)]:
        g = graphs.build(name, size)
        out = I.run_graph(g, gen.make_weights(g), gen.make_input(g), keep={g.n_ops - 1})
        y = out[g.n_ops - 1]
        assert np.isfinite(y).all() and np.abs(y).max() > 0


def test_add_hand_computed():
    """add (oracle/infer.py run_op 'add'): y = act(sum_i agg_i x_i), agg_i = 1
    when the op carries no weights.  Values worked by hand."""
    g = graphs.GraphSpec("add", 1, 1, 2)
    x0 = g.input()
    plain = g.add([x0, x0, x0], relu=0)          # 3 x
    plain_r = g.add([x0, x0], relu=1)            # relu(2 x)
    weighted = g.add([x0, x0], relu=0, agg=1)    # (1/2 + 1/2) x = x (gen: agg = 1/n)
    op = {o.id: o for o in g.ops}
    x = np.array([[[-1.5, 2.0]]])
    assert np.array_equal(I.run_op(op[plain], [x, x, x], {}), [[[-4.5, 6.0]]])
    assert np.array_equal(I.run_op(op[plain_r], [x, x], {}), [[[0.0, 4.0]]])
    w = {"agg": np.array([0.25, 0.75], dtype=np.float32)}
    y = I.run_op(op[weighted], [x, 2 * x], w)    # 0.25 x + 1.5 x = 1.75 x
    assert np.array_equal(y, [[[-2.625, 3.5]]])
    op[weighted].relu = 1
    assert np.array_equal(I.run_op(op[weighted], [x, 2 * x], w), [[[0.0, 3.5]]])
    # a single-input ReLU add and the input order (slot order) of weights
    one = g.add([x0], relu=1)
    assert np.array_equal(I.run_op({o.id: o for o in g.ops}[one], [x], {}), [[[0.0, 2.0]]])
    w2 = {"agg": np.array([1.0, -3.0], dtype=np.float32)}
    op[weighted].relu = 0
    assert np.array_equal(I.run_op(op[weighted], [x, 0 * x + 1.0], w2), [[[-4.5, -1.0]]])


@pytest.mark.parametrize("n_in,agg,act", [(2, 0, 0), (2, 0, 1), (5, 1, 1), (4, 1, 0)])
def test_add_vs_torch_in_graph(n_in, agg, act):
    """The add branch as run_graph reaches it (edge slots, gen's aggregation
    weights), against torch fp64: relu(sum_i a_i x_i) by torch.stack /
    tensordot, a_i = gen's agg weights or 1."""
    g = graphs.GraphSpec("addg", 3, 7, 6)
    x0 = g.input()
    ins = [g.conv(x0, 5, 3, p=1, relu=0) for _ in range(n_in)]
    s = g.add(ins[::-1], relu=act, agg=agg)       # reversed: slot order != id order
    W = gen.make_weights(g)
    x = gen.make_input(g)
    out = I.run_graph(g, W, x)
    t = torch.stack([torch.from_numpy(out[i]) for i in ins[::-1]])
    a = torch.from_numpy(W[s]["agg"].astype(np.float64)) if agg else torch.ones(n_in, dtype=torch.float64)
    ref = torch.tensordot(a, t, dims=([0], [0]))
    if act:
        ref = F.relu(ref)
    np.testing.assert_allclose(out[s], ref.numpy(), rtol=1e-13, atol=1e-13)
    if agg:  # gen's add weights are 1/n: the aggregation is the mean
        np.testing.assert_allclose(W[s]["agg"].astype(np.float64).sum(), 1.0, rtol=1e-6)


def test_identity_is_a_copy():
    g = graphs.GraphSpec("id", 4, 5, 5)
    x0 = g.input()
    c = g.conv(x0, 6, 3, p=1)
    i = g.identity(c)
    g.add([i, c], relu=0)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    out = I.run_graph(g, W, x)
    assert np.array_equal(out[i], out[c])
    np.testing.assert_array_equal(out[g.n_ops - 1], 2 * out[c])
    y = I.run_op(g.ops[i], [out[c]], {})
    y += 1.0                                       # a copy, not a view of the input
    assert np.array_equal(out[i], out[c])


def test_conv_pre_relu_vs_torch():
    """conv with pre_relu (NASNet's ReLU -> conv -> BN): torch fp64 relu then conv2d."""
    g = graphs.GraphSpec("pr", 5, 9, 11)
    x0 = g.input()
    c = g.conv(x0, 7, 3, s=2, p=1, relu=0, pre_relu=1)
    W = gen.make_weights(g)
    x = gen.make_input(g) - 0.5            # negative inputs: the pre-ReLU matters
    out = I.run_graph(g, W, x)
    t = F.relu(torch.from_numpy(x.astype(np.float64)))
    ref = F.conv2d(t, torch.from_numpy(W[c]["weight"].astype(np.float64)), stride=2, padding=1)[0]
    ref = ref * torch.from_numpy(W[c]["scale"].astype(np.float64))[:, None, None] + \
        torch.from_numpy(W[c]["shift"].astype(np.float64))[:, None, None]
    np.testing.assert_allclose(out[c], ref.numpy(), rtol=1e-12, atol=1e-12)
    assert not np.allclose(out[c], I.conv2d(x[0].astype(np.float64), W[c]["weight"].astype(np.float64), 2, 2, 1, 1)
                           * W[c]["scale"][:, None, None] + W[c]["shift"][:, None, None])


@pytest.mark.parametrize("H", [12, 13])
def test_nasnet_factorized_reduction_vs_reference_formulation(H):
    """The factorized reduction as the public NASNet-A code writes it (ReLU;
    path 1 = AvgPool(1, stride 2) -> 1x1 conv; path 2 = pad (0,1,0,1), drop
    the first row / column, AvgPool(1, stride 2) -> 1x1 conv; concat) against
    this IR's reading: a stride-2 1x1 conv and a 3x3 / stride 2 / pad 1 conv
    whose only non-zero tap is (2, 2) (workloads/graphs.py _nas_factorized),
    even and odd input sizes."""
    g = graphs.GraphSpec("fr", 6, H, H)
    x0 = g.input()
    cat = graphs._nas_factorized(g, x0, 8, "fr")
    p1, p2 = g.preds(cat)
    W = gen.make_weights(g)
    x = gen.make_input(g) - 0.5
    out = I.run_graph(g, W, x)
    t = F.relu(torch.from_numpy(x.astype(np.float64)))
    a = F.avg_pool2d(t, 1, stride=2, count_include_pad=False)
    w1 = torch.from_numpy(W[p1]["weight"].astype(np.float64))
    y1 = F.conv2d(a, w1)
    b = F.pad(t, (0, 1, 0, 1))[:, :, 1:, 1:]
    b = F.avg_pool2d(b, 1, stride=2, count_include_pad=False)
    w2 = torch.from_numpy(W[p2]["weight"][:, :, 2, 2].astype(np.float64))[:, :, None, None]
    y2 = F.conv2d(b, w2)

    def bn(y, v):
        return y * torch.from_numpy(W[v]["scale"].astype(np.float64))[None, :, None, None] + \
            torch.from_numpy(W[v]["shift"].astype(np.float64))[None, :, None, None]
    ref = torch.cat([bn(y1, p1), bn(y2, p2)], 1)[0].numpy()
    assert out[cat].shape == ref.shape
    np.testing.assert_allclose(out[cat], ref, rtol=1e-12, atol=1e-12)
    # the single-tap conv's other taps are zero in the generated weights
    wt = W[p2]["weight"].copy()
    wt[:, :, 2, 2] = 0
    assert not wt.any()
