"""DAG-CNN workload builders (structure only -- no arithmetic of the method).

These builders are *workload data*: they emit the operator list and the edge
list of the computation graph G = (V, E) of PAPER.md §III-A: "each
vertex v in V represents an operator, such as convolution, pooling, and linear
operators, and each edge e = (u, v) in E indicates an operator dependency,
i.e., a tensor that is the output of operator u and the input of operator v."

Both the CPU oracle (``oracle/``) and the CUDA path (through the C-ABI) consume
the same lists; neither side's arithmetic lives here.  The only bookkeeping is
the output *channel count* of each op, needed to size the seeded weights
(``workloads/gen.py``).  Spatial shapes are inferred independently by the
oracle (by computing) and by the C++ graph IR.

Operator granularity follows SURVEY.md §8(c) C20: conv+BN+ReLU is one op,
each pool is one op, one concat per block, plus an input placeholder op.

Op kinds (string -> C-ABI enum in the binding):
  input, conv, sepconv, maxpool, avgpool, gap, concat, add, linear, identity
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Tuple

KINDS = ("input", "conv", "sepconv", "maxpool", "avgpool", "gap", "concat",
         "add", "linear", "identity")


@dataclass
class OpSpec:
    id: int
    kind: str
    name: str
    in_c: int = 0          # input channels (conv / sepconv / linear weight sizing)
    out_c: int = 0
    kh: int = 1
    kw: int = 1
    sh: int = 1
    sw: int = 1
    ph: int = 0
    pw: int = 0
    dh: int = 1
    dw: int = 1
    relu: int = 0          # ReLU after (BN-folded) affine / after sum
    pre_relu: int = 0      # sepconv: ReLU applied to the (aggregated) input first
    ceil_mode: int = 0     # pools
    count_include_pad: int = 1  # avgpool
    agg: int = 0           # add / sepconv: weighted aggregation of the inputs
    reps: int = 1          # sepconv: (ReLU -> dw -> pw -> BN) repetitions
    n_in: int = 0
    tap: Optional[Tuple[int, int]] = None  # conv: the only non-zero kernel tap (weights sized by in_c)


@dataclass
class GraphSpec:
    name: str
    in_c: int
    in_h: int
    in_w: int
    ops: List[OpSpec] = field(default_factory=list)
    edges: List[Tuple[int, int, int]] = field(default_factory=list)  # (src, dst, slot)

    # ------------------------------------------------------------------ build
    def _add(self, kind: str, inputs: List[int], name: str = "", **p) -> int:
        oid = len(self.ops)
        op = OpSpec(id=oid, kind=kind, name=name or f"{kind}{oid}", **p)
        op.n_in = len(inputs)
        for slot, src in enumerate(inputs):
            assert 0 <= src < oid, "builders emit ops in topological order"
            self.edges.append((src, oid, slot))
        self.ops.append(op)
        return oid

    def chan(self, oid: int) -> int:
        return self.ops[oid].out_c

    def input(self) -> int:
        return self._add("input", [], name="input", out_c=self.in_c)

    def conv(self, x: int, out_c: int, k, s=1, p=0, relu=1, name="", pre_relu=0, tap=None) -> int:
        """conv (+ folded BN) (+ ReLU); pre_relu: ReLU applied to the input
        first (NASNet's ReLU -> conv -> BN); tap: a single-tap conv (a shifted,
        strided 1x1 conv: the other taps' weights are zero, workloads/gen.py)."""
        kh, kw = (k, k) if isinstance(k, int) else k
        sh, sw = (s, s) if isinstance(s, int) else s
        ph, pw = (p, p) if isinstance(p, int) else p
        return self._add("conv", [x], name, in_c=self.chan(x), out_c=out_c,
                         kh=kh, kw=kw, sh=sh, sw=sw, ph=ph, pw=pw, relu=relu, pre_relu=pre_relu, tap=tap)

    def sepconv(self, xs: List[int], out_c: int, k: int, s: int = 1,
                pre_relu=1, relu=0, agg=None, reps=1, name="") -> int:
        cin = self.chan(xs[0])
        assert all(self.chan(x) == cin for x in xs)
        if agg is None:
            agg = 1 if len(xs) > 1 else 0
        return self._add("sepconv", list(xs), name, in_c=cin, out_c=out_c,
                         kh=k, kw=k, sh=s, sw=s, ph=k // 2, pw=k // 2,
                         pre_relu=pre_relu, relu=relu, agg=agg, reps=reps)

    def maxpool(self, x: int, k: int, s: int, p: int = 0, ceil_mode=0, name="") -> int:
        return self._add("maxpool", [x], name, in_c=self.chan(x), out_c=self.chan(x),
                         kh=k, kw=k, sh=s, sw=s, ph=p, pw=p, ceil_mode=ceil_mode)

    def avgpool(self, x: int, k: int, s: int, p: int = 0, count_include_pad=1,
                ceil_mode=0, name="") -> int:
        return self._add("avgpool", [x], name, in_c=self.chan(x), out_c=self.chan(x),
                         kh=k, kw=k, sh=s, sw=s, ph=p, pw=p,
                         count_include_pad=count_include_pad, ceil_mode=ceil_mode)

    def gap(self, x: int, name="") -> int:
        return self._add("gap", [x], name, in_c=self.chan(x), out_c=self.chan(x))

    def concat(self, xs: List[int], name="") -> int:
        return self._add("concat", list(xs), name, out_c=sum(self.chan(x) for x in xs))

    def add(self, xs: List[int], relu=0, agg=0, name="") -> int:
        c = self.chan(xs[0])
        assert all(self.chan(x) == c for x in xs)
        return self._add("add", list(xs), name, in_c=c, out_c=c, relu=relu, agg=agg)

    def linear(self, x: int, out_c: int, name="") -> int:
        return self._add("linear", [x], name, in_c=self.chan(x), out_c=out_c)

    def identity(self, x: int, name="") -> int:
        return self._add("identity", [x], name, in_c=self.chan(x), out_c=self.chan(x))

    # ------------------------------------------------------------------ query
    @property
    def n_ops(self) -> int:
        return len(self.ops)

    @property
    def n_edges(self) -> int:
        return len(self.edges)

    def preds(self, v: int) -> List[int]:
        return [s for (s, d, _) in sorted(self.edges, key=lambda e: (e[1], e[2])) if d == v]

    def sinks(self) -> List[int]:
        srcs = {s for (s, _, _) in self.edges}
        return [o.id for o in self.ops if o.id not in srcs]


# ============================================================================
# tiny: the Fig. 4 topology as conv ops on 1x64x56x56
# ============================================================================
def tiny(h: int = 56, w: int = 56, c: int = 64) -> GraphSpec:
    """Fig. 4 DAG: e1=v1->v2, e2=v1->v3, e3=v2->v4, e4=v3->v5, e5=v4->v6,
    e6=v5->v6, e7=v5->v7, e8=v6->v8, e9=v7->v8, plus an input
    placeholder feeding v1."""
    g = GraphSpec("tiny", c, h, w)
    x = g.input()
    v1 = g.conv(x, c, 3, p=1, name="v1")
    v2 = g.conv(v1, c, 3, p=1, name="v2")
    v3 = g.conv(v1, c, 1, name="v3")
    v4 = g.conv(v2, c, 3, p=1, name="v4")
    v5 = g.conv(v3, c, 3, p=1, name="v5")
    v6 = g.add([v4, v5], relu=1, name="v6")
    v7 = g.conv(v5, c, 3, p=1, name="v7")
    g.concat([v6, v7], name="v8")
    return g


# ============================================================================
# Inception-v3 (Szegedy et al. [16]); torchvision module naming
# ============================================================================
def _inc_a(g, x, pool_features, pfx):
    b1 = g.conv(x, 64, 1, name=f"{pfx}.branch1x1")
    b5 = g.conv(x, 48, 1, name=f"{pfx}.branch5x5_1")
    b5 = g.conv(b5, 64, 5, p=2, name=f"{pfx}.branch5x5_2")
    b3 = g.conv(x, 64, 1, name=f"{pfx}.branch3x3dbl_1")
    b3 = g.conv(b3, 96, 3, p=1, name=f"{pfx}.branch3x3dbl_2")
    b3 = g.conv(b3, 96, 3, p=1, name=f"{pfx}.branch3x3dbl_3")
    bp = g.avgpool(x, 3, 1, 1, name=f"{pfx}.avg_pool")
    bp = g.conv(bp, pool_features, 1, name=f"{pfx}.branch_pool")
    return g.concat([b1, b5, b3, bp], name=f"{pfx}.concat")


def _inc_b(g, x, pfx):
    b3 = g.conv(x, 384, 3, s=2, name=f"{pfx}.branch3x3")
    bd = g.conv(x, 64, 1, name=f"{pfx}.branch3x3dbl_1")
    bd = g.conv(bd, 96, 3, p=1, name=f"{pfx}.branch3x3dbl_2")
    bd = g.conv(bd, 96, 3, s=2, name=f"{pfx}.branch3x3dbl_3")
    bp = g.maxpool(x, 3, 2, name=f"{pfx}.max_pool")
    return g.concat([b3, bd, bp], name=f"{pfx}.concat")


def _inc_c(g, x, c7, pfx):
    b1 = g.conv(x, 192, 1, name=f"{pfx}.branch1x1")
    b7 = g.conv(x, c7, 1, name=f"{pfx}.branch7x7_1")
    b7 = g.conv(b7, c7, (1, 7), p=(0, 3), name=f"{pfx}.branch7x7_2")
    b7 = g.conv(b7, 192, (7, 1), p=(3, 0), name=f"{pfx}.branch7x7_3")
    bd = g.conv(x, c7, 1, name=f"{pfx}.branch7x7dbl_1")
    bd = g.conv(bd, c7, (7, 1), p=(3, 0), name=f"{pfx}.branch7x7dbl_2")
    bd = g.conv(bd, c7, (1, 7), p=(0, 3), name=f"{pfx}.branch7x7dbl_3")
    bd = g.conv(bd, c7, (7, 1), p=(3, 0), name=f"{pfx}.branch7x7dbl_4")
    bd = g.conv(bd, 192, (1, 7), p=(0, 3), name=f"{pfx}.branch7x7dbl_5")
    bp = g.avgpool(x, 3, 1, 1, name=f"{pfx}.avg_pool")
    bp = g.conv(bp, 192, 1, name=f"{pfx}.branch_pool")
    return g.concat([b1, b7, bd, bp], name=f"{pfx}.concat")


def _inc_d(g, x, pfx):
    b3 = g.conv(x, 192, 1, name=f"{pfx}.branch3x3_1")
    b3 = g.conv(b3, 320, 3, s=2, name=f"{pfx}.branch3x3_2")
    b7 = g.conv(x, 192, 1, name=f"{pfx}.branch7x7x3_1")
    b7 = g.conv(b7, 192, (1, 7), p=(0, 3), name=f"{pfx}.branch7x7x3_2")
    b7 = g.conv(b7, 192, (7, 1), p=(3, 0), name=f"{pfx}.branch7x7x3_3")
    b7 = g.conv(b7, 192, 3, s=2, name=f"{pfx}.branch7x7x3_4")
    bp = g.maxpool(x, 3, 2, name=f"{pfx}.max_pool")
    return g.concat([b3, b7, bp], name=f"{pfx}.concat")


def _inc_e(g, x, pfx):
    b1 = g.conv(x, 320, 1, name=f"{pfx}.branch1x1")
    b3 = g.conv(x, 384, 1, name=f"{pfx}.branch3x3_1")
    b3a = g.conv(b3, 384, (1, 3), p=(0, 1), name=f"{pfx}.branch3x3_2a")
    b3b = g.conv(b3, 384, (3, 1), p=(1, 0), name=f"{pfx}.branch3x3_2b")
    bd = g.conv(x, 448, 1, name=f"{pfx}.branch3x3dbl_1")
    bd = g.conv(bd, 384, 3, p=1, name=f"{pfx}.branch3x3dbl_2")
    bda = g.conv(bd, 384, (1, 3), p=(0, 1), name=f"{pfx}.branch3x3dbl_3a")
    bdb = g.conv(bd, 384, (3, 1), p=(1, 0), name=f"{pfx}.branch3x3dbl_3b")
    bp = g.avgpool(x, 3, 1, 1, name=f"{pfx}.avg_pool")
    bp = g.conv(bp, 192, 1, name=f"{pfx}.branch_pool")
    # InceptionE's inner concats are flattened into the block concat (C20)
    return g.concat([b1, b3a, b3b, bda, bdb, bp], name=f"{pfx}.concat")


def inception_v3(h: int = 299, w: Optional[int] = None, head: bool = True) -> GraphSpec:
    """Inception-v3, batch 1.  Core = 119 ops / 153 edges counting the
    input placeholder; ``head`` adds GAP + FC(2048->1000) (121 / 155)."""
    w = h if w is None else w
    g = GraphSpec(f"inception_v3_{h}", 3, h, w)
    x = g.input()
    x = g.conv(x, 32, 3, s=2, name="Conv2d_1a_3x3")
    x = g.conv(x, 32, 3, name="Conv2d_2a_3x3")
    x = g.conv(x, 64, 3, p=1, name="Conv2d_2b_3x3")
    x = g.maxpool(x, 3, 2, name="maxpool1")
    x = g.conv(x, 80, 1, name="Conv2d_3b_1x1")
    x = g.conv(x, 192, 3, name="Conv2d_4a_3x3")
    x = g.maxpool(x, 3, 2, name="maxpool2")
    x = _inc_a(g, x, 32, "Mixed_5b")
    x = _inc_a(g, x, 64, "Mixed_5c")
    x = _inc_a(g, x, 64, "Mixed_5d")
    x = _inc_b(g, x, "Mixed_6a")
    x = _inc_c(g, x, 128, "Mixed_6b")
    x = _inc_c(g, x, 160, "Mixed_6c")
    x = _inc_c(g, x, 160, "Mixed_6d")
    x = _inc_c(g, x, 192, "Mixed_6e")
    x = _inc_d(g, x, "Mixed_7a")
    x = _inc_e(g, x, "Mixed_7b")
    x = _inc_e(g, x, "Mixed_7c")
    if head:
        x = g.gap(x, name="avgpool")
        g.linear(x, 1000, name="fc")
    return g


# ============================================================================
# SqueezeNet 1.0 (north-star addition, BASELINE.json configs[4])
# ============================================================================
def _fire(g, x, sq, e1, e3, pfx):
    s = g.conv(x, sq, 1, name=f"{pfx}.squeeze")
    a = g.conv(s, e1, 1, name=f"{pfx}.expand1x1")
    b = g.conv(s, e3, 3, p=1, name=f"{pfx}.expand3x3")
    return g.concat([a, b], name=f"{pfx}.concat")


def squeezenet(h: int = 224, w: Optional[int] = None) -> GraphSpec:
    """SqueezeNet 1.0 (torchvision layout; features.N indices in names)."""
    w = h if w is None else w
    g = GraphSpec(f"squeezenet_{h}", 3, h, w)
    x = g.input()
    x = g.conv(x, 96, 7, s=2, name="features.0")
    x = g.maxpool(x, 3, 2, ceil_mode=1, name="features.2")
    x = _fire(g, x, 16, 64, 64, "features.3")
    x = _fire(g, x, 16, 64, 64, "features.4")
    x = _fire(g, x, 32, 128, 128, "features.5")
    x = g.maxpool(x, 3, 2, ceil_mode=1, name="features.6")
    x = _fire(g, x, 32, 128, 128, "features.7")
    x = _fire(g, x, 48, 192, 192, "features.8")
    x = _fire(g, x, 48, 192, 192, "features.9")
    x = _fire(g, x, 64, 256, 256, "features.10")
    x = g.maxpool(x, 3, 2, ceil_mode=1, name="features.11")
    x = _fire(g, x, 64, 256, 256, "features.12")
    x = g.conv(x, 1000, 1, name="classifier.1")
    g.gap(x, name="classifier.3")
    return g


# ============================================================================
# RandWire-WS, small regime (Xie et al.; IOS's benchmark set) -- north-star add
# ============================================================================
# WS(N=32, K=4, P=0.75) graphs, generated once with
#   networkx.connected_watts_strogatz_graph(32, 4, 0.75, seed=s), s = 0, 1, 2
# and oriented low id -> high id.  Frozen in workloads/randwire_ws_edges.json
# (regenerated by workloads/make_randwire_edges.py) so a networkx change
# cannot alter the workload.
def _randwire_edges() -> List[List[Tuple[int, int]]]:
    import json
    import os
    p = os.path.join(os.path.dirname(__file__), "randwire_ws_edges.json")
    with open(p) as f:
        return [[tuple(e) for e in s] for s in json.load(f)["stages"]]


def _randwire_stage(g, x, edges, n, out_c, pfx):
    preds: Dict[int, List[int]] = {i: [] for i in range(n)}
    succs: Dict[int, List[int]] = {i: [] for i in range(n)}
    for (a, b) in edges:
        preds[b].append(a)
        succs[a].append(b)
    node_op: Dict[int, int] = {}
    for i in range(n):  # ids are a topological order (edges go low -> high)
        if not preds[i]:
            # input node: ReLU -> sepconv stride 2 on the stage input
            node_op[i] = g.sepconv([x], out_c, 3, s=2, pre_relu=1, name=f"{pfx}.node{i}")
        else:
            ins = [node_op[j] for j in sorted(preds[i])]
            node_op[i] = g.sepconv(ins, out_c, 3, s=1, pre_relu=1,
                                   agg=1 if len(ins) > 1 else 0, name=f"{pfx}.node{i}")
    outs = [node_op[i] for i in range(n) if not succs[i]]
    if len(outs) == 1:
        return outs[0]
    return g.add(outs, agg=1, name=f"{pfx}.out")  # unweighted mean: agg weights 1/k


def randwire_ws(h: int = 224, w: Optional[int] = None, c: int = 78) -> GraphSpec:
    """RandWire-WS small regime: conv1 (3x3 s2, C/2) -> conv2 (3x3 s2, C) ->
    three random-wiring stages (N=32 each; C, 2C, 4C) -> 1x1 conv 1280 ->
    GAP -> FC 1000.  Node = weighted aggregation -> ReLU -> sepconv 3x3 -> BN."""
    w = h if w is None else w
    g = GraphSpec(f"randwire_ws_{h}", 3, h, w)
    stages = _randwire_edges()
    x = g.input()
    x = g.conv(x, c // 2, 3, s=2, p=1, relu=1, name="conv1")   # conv1 -> BN (-> conv2's ReLU)
    x = g.conv(x, c, 3, s=2, p=1, relu=0, name="conv2")        # ReLU-conv-BN
    for si, (edges, mult) in enumerate(zip(stages, (1, 2, 4))):
        x = _randwire_stage(g, x, edges, 32, c * mult, f"stage{si + 3}")
    x = g.conv(x, 1280, 1, relu=1, name="classifier.conv")
    x = g.gap(x, name="gap")
    g.linear(x, 1000, name="fc")
    return g


# ============================================================================
# NASNet-A large (north star: "NASNet-A large"; P:297 counts 374 ops / 576 deps)
# ============================================================================
# Zoph et al. [17] cells as in the public NASNet-A-large (N = 6, penultimate
# filters 4032, F = 168): every cell input passes ReLU -> 1x1 conv -> BN
# ("fit"); a previous-cell input at twice the resolution passes the factorized
# reduction (ReLU -> two stride-2 1x1 convs, the second on the input shifted by
# one pixel -> concat -> BN); separable branches are (ReLU -> sep kxk -> BN)
# twice; the network ends ReLU -> GAP -> FC.
def _nas_sep(g, x, c, k, s, pfx):
    """NASNet separable block: (ReLU -> sep kxk -> BN) twice, the first with
    stride s -- one operator (IOS-style sequential block)."""
    return g.sepconv([x], c, k, s=s, pre_relu=1, reps=2, name=pfx)


def _nas_fit(g, x, c, pfx):
    """ReLU -> 1x1 conv -> BN."""
    return g.conv(x, c, 1, relu=0, pre_relu=1, name=pfx)


def _nas_factorized(g, x, c, pfx):
    """Factorized reduction of a 2x-resolution input to c channels: path 1 =
    ReLU -> 1x1 conv stride 2 (pixels 2p, 2q); path 2 = the same on the input
    shifted by one pixel (pixels 2p+1, 2q+1, zero past the edge) -- a 3x3 /
    stride 2 / pad 1 conv whose only non-zero tap is (2, 2); concat; the BN is
    folded into each path's conv (per output channel)."""
    a = g.conv(x, c // 2, 1, s=2, relu=0, pre_relu=1, name=f"{pfx}.path1")
    b = g.conv(x, c - c // 2, 3, s=2, p=1, relu=0, pre_relu=1, tap=(2, 2), name=f"{pfx}.path2")
    return g.concat([a, b], name=f"{pfx}.cat")


def _nas_normal(g, h, h_prev, c, pfx, first=False):
    """NASNet-A normal cell (Fig. 4 left of [17]); FirstCell when h_prev has
    twice h's resolution (factorized reduction of h_prev).  Output = concat of
    the adjusted h_prev and the 5 block outputs."""
    x = _nas_fit(g, h, c, f"{pfx}.fit_h")
    p = _nas_factorized(g, h_prev, c, f"{pfx}.fact_prev") if first else _nas_fit(g, h_prev, c, f"{pfx}.fit_prev")
    b0 = g.add([_nas_sep(g, x, c, 5, 1, f"{pfx}.b0l"), _nas_sep(g, p, c, 3, 1, f"{pfx}.b0r")],
               name=f"{pfx}.b0")
    b1 = g.add([_nas_sep(g, p, c, 5, 1, f"{pfx}.b1l"), _nas_sep(g, p, c, 3, 1, f"{pfx}.b1r")],
               name=f"{pfx}.b1")
    b2 = g.add([g.avgpool(x, 3, 1, 1, count_include_pad=0, name=f"{pfx}.b2l"), p], name=f"{pfx}.b2")
    b3 = g.add([g.avgpool(p, 3, 1, 1, count_include_pad=0, name=f"{pfx}.b3l"),
                g.avgpool(p, 3, 1, 1, count_include_pad=0, name=f"{pfx}.b3r")], name=f"{pfx}.b3")
    b4 = g.add([_nas_sep(g, x, c, 3, 1, f"{pfx}.b4l"), x], name=f"{pfx}.b4")
    return g.concat([p, b0, b1, b2, b3, b4], name=f"{pfx}.concat")


def _nas_reduction(g, x, p, c, pfx):
    """NASNet-A reduction cell (Fig. 4 right of [17]) on the adjusted inputs
    x (from h) and p (from h_prev)."""
    b0 = g.add([_nas_sep(g, x, c, 5, 2, f"{pfx}.b0l"), _nas_sep(g, p, c, 7, 2, f"{pfx}.b0r")],
               name=f"{pfx}.b0")
    b1 = g.add([g.maxpool(x, 3, 2, 1, name=f"{pfx}.b1l"), _nas_sep(g, p, c, 7, 2, f"{pfx}.b1r")],
               name=f"{pfx}.b1")
    b2 = g.add([g.avgpool(x, 3, 2, 1, count_include_pad=0, name=f"{pfx}.b2l"),
                _nas_sep(g, p, c, 5, 2, f"{pfx}.b2r")], name=f"{pfx}.b2")
    b3 = g.add([g.avgpool(b0, 3, 1, 1, count_include_pad=0, name=f"{pfx}.b3l"), b1], name=f"{pfx}.b3")
    b4 = g.add([_nas_sep(g, b0, c, 3, 1, f"{pfx}.b4l"), g.maxpool(x, 3, 2, 1, name=f"{pfx}.b4r")],
               name=f"{pfx}.b4")
    return g.concat([b1, b2, b3, b4], name=f"{pfx}.concat")


def nasnet_a_large(h: int = 331, w: Optional[int] = None, n: int = 6, f: int = 168,
                   stem_c: int = 96) -> GraphSpec:
    """NASNet-A large (N = 6 normal cells per stack, F = 168): stem conv 3x3 s2
    (+BN), cell_stem_0 (its second input is the raw stem output, whose
    separable branches map 96 -> F/4 channels), cell_stem_1 (factorized
    reduction of the stem output), 3 stacks of N normal cells (the first of
    each a FirstCell) separated by two reduction cells, ReLU -> GAP -> FC."""
    w = h if w is None else w
    g = GraphSpec(f"nasnet_a_large_{h}", 3, h, w)
    x = g.input()
    stem = g.conv(x, stem_c, 3, s=2, relu=0, name="conv0")
    # cell_stem_0: x1 = fit(stem); the "left" separable branches read the raw stem
    c = f // 4
    cur = _nas_reduction(g, _nas_fit(g, stem, c, "cell_stem_0.fit_h"), stem, c, "cell_stem_0")
    # cell_stem_1: fit(cell_stem_0), factorized reduction of the stem output
    c = f // 2
    nxt = _nas_reduction(g, _nas_fit(g, cur, c, "cell_stem_1.fit_h"), _nas_factorized(g, stem, c, "cell_stem_1.fact_prev"),
                         c, "cell_stem_1")
    prev, cur = cur, nxt
    c = f
    for stack in range(3):
        for i in range(n):
            nxt = _nas_normal(g, cur, prev, c, f"cell_{stack}_{i}", first=(i == 0))
            prev, cur = cur, nxt
        if stack < 2:
            c *= 2
            r = _nas_reduction(g, _nas_fit(g, cur, c, f"reduction_cell_{stack}.fit_h"),
                               _nas_fit(g, prev, c, f"reduction_cell_{stack}.fit_prev"), c,
                               f"reduction_cell_{stack}")
            prev, cur = cur, r
    x = g.add([cur], relu=1, name="relu")
    x = g.gap(x, name="avgpool")
    g.linear(x, 1000, name="last_linear")
    return g


BUILDERS = {
    "tiny": tiny,
    "inception_v3": inception_v3,
    "squeezenet": squeezenet,
    "randwire_ws": randwire_ws,
    "nasnet_a_large": nasnet_a_large,
}


def build(name: str, size: Optional[int] = None) -> GraphSpec:
    fn = BUILDERS[name]
    if name == "tiny":
        return fn() if size is None else fn(size, size)
    return fn() if size is None else fn(size)
