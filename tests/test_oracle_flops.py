"""Pins for graph.flops (reading R1: the FLOP counts Alg. 1's Overhead compares,
P:L219): hand-counted values for every operator kind on a tiny graph, written out
as plain numbers here (not by re-evaluating the formulas), plus the Overhead
decision they drive on a case where kh*kw matters."""
import pytest

import oracle
import workloads as W
from oracle.graph import Graph, Node, flops


def _g(nodes):
    return Graph(nodes=nodes, output=nodes[-1].id, batch=2, dtype="f32", orig_flops={},
                 nodes_by_id={n.id: n for n in nodes})


def test_flops_hand_counts_per_operator():
    # x: 2 images of 4 x 6 x 6
    x = Node(0, "input", [], C=4, H=6, W=6)
    conv = Node(1, "conv", [0], kh=3, kw=3, sh=1, sw=1, ph=1, pw=1, C=8, H=6, W=6)     # 3x3, 4 -> 8
    dw = Node(2, "conv", [1], kh=3, kw=1, sh=2, sw=1, ph=1, pw=0, groups=8, C=8, H=3, W=6)  # depthwise 3x1 s(2,1)
    bn = Node(3, "bn", [2], C=8, H=3, W=6)
    relu = Node(4, "relu", [3], C=8, H=3, W=6)
    silu = Node(5, "silu", [4], C=8, H=3, W=6)
    add = Node(6, "add", [4, 5, 3], C=8, H=3, W=6)
    mp = Node(7, "maxpool", [6], kh=3, kw=3, sh=2, sw=2, ph=1, pw=1, C=8, H=2, W=3)
    ap = Node(8, "avgpool", [6], kh=2, kw=2, sh=2, sw=2, C=8, H=1, W=3)
    cat = Node(9, "concat", [7, 7], C=16, H=2, W=3)
    gap = Node(10, "gap", [9], C=16, H=1, W=1)
    lin = Node(11, "linear", [10], C=10, H=1, W=1)
    g = _g([x, conv, dw, bn, relu, silu, add, mp, ap, cat, gap, lin])
    # conv: 2 img * 36 px * 8 out * (4 in * 9 taps) * 2 = 41472
    assert flops(g, conv) == 41472
    # depthwise: 2 * 18 px * 8 ch * (1 * 3 taps) * 2 = 1728
    assert flops(g, dw) == 1728
    # bn: 2 per element, 2*8*3*6 = 288 elements
    assert flops(g, bn) == 576
    assert flops(g, relu) == 288
    assert flops(g, silu) == 1152            # 4 per element
    assert flops(g, add) == 576              # 3 inputs: 2 adds per element
    assert flops(g, mp) == 2 * 8 * 6 * 9     # k^2 per output element: 864
    assert flops(g, ap) == 2 * 8 * 3 * 4     # 192
    assert flops(g, cat) == 0
    assert flops(g, gap) == 2 * 16 * 6       # one add per input element: 192
    assert flops(g, lin) == 2 * 16 * 10 * 2  # 640
    # transposed conv 2x2 / stride 2, 4 -> 6 channels on a 3 x 5 input (output 6 x 10): every
    # input pixel meets every weight once: 2 img * 15 px * 4 in * 6 out * 4 taps * 2 = 5760
    xt = Node(12, "input", [], C=4, H=3, W=5)
    ct = Node(13, "convt", [12], kh=2, kw=2, sh=2, sw=2, ph=0, pw=0, C=6, H=6, W=10)
    assert flops(_g([xt, ct]), ct) == 5760


def test_overhead_uses_the_kernel_window():
    """A 3x3 conv 4 -> 16 decomposed with ranks (4, 8) (fconv omitted): copying its lconv
    (2*8*16 per pixel) costs less than the original 3x3 conv (2*4*16*9 per pixel), so the
    skip is optimized; with a 1x1 original the same copy would cost more (the test in
    test_oracle_rewrite.py) -- the decision depends on the kh*kw term of R1."""
    g = W.models._G("overhead3", 1, 6, 6, 4, "f32", 9, rank=lambda c: 4 if c == 4 else 8)
    a = g.relu(g.conv(0, 16, 3, 1, 1, name="up"), "relu")
    b = g.relu(g.conv(a, 16, 3, 1, 1, name="mid"), "relu2")
    g.add([b, a], "add")
    pl = oracle.plan(g.m)
    assert pl.log[0][0] == "skip-optimized"
