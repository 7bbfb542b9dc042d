"""Decomposed IR and decomposition expansion (oracle step O1).

PAPER.md P:L83-91 (Fig. 2): a decomposed convolution is a sequence
  fconv (1x1, C -> C1, "reduce")  ->  core convolution(s)  ->  lconv (1x1, C2 -> C', "restore");
the first and last factors are consistent across decomposition methods, the
core differs.  Eq. (2) gives the factor shapes C*C1, C1*C2*K^2,
C2*C' for Tucker.

Readings:
  * R16 (Fig. 1 lost): CP is realised Lebedev-style as
      fconv (C_in -> R) -> depthwise K x 1 (stride (s,1), pad (p,0))
      -> depthwise 1 x K (stride (1,s), pad (0,p)) -> lconv (R -> C_out).
  * O1: stride and padding sit on the core; the original bias sits on the
    lconv (on the core when the lconv is absent).  A Tucker-2 factor is absent
    when its rank equals the mode size (the builder passes None).
  * R14: SIZE(v) = N * C * H * W * sizeof(plan dtype) bytes.
  * R1: FLOP counts used by Overhead.
"""
from __future__ import annotations

from dataclasses import dataclass, field, replace
from typing import Optional

import numpy as np

DTYPE_BYTES = {"f32": 4, "bf16": 2}


@dataclass
class Node:
    id: int
    op: str                       # input conv bn relu silu add concat maxpool avgpool gap linear
    inputs: list
    role: str = ""                # fconv | core | lconv | ""
    orig: int = -1                # index of the original layer
    name: str = ""
    kh: int = 1
    kw: int = 1
    sh: int = 1
    sw: int = 1
    ph: int = 0
    pw: int = 0
    groups: int = 1
    C: int = 0                    # per-image output shape (C, H, W)
    H: int = 0
    W: int = 0
    weight: Optional[np.ndarray] = None
    bias: Optional[np.ndarray] = None
    bn: Optional[tuple] = None    # (gamma, beta, mean, var, eps)
    copy_of: int = -1             # for COPY(l.list) clones: the id of the original node

    def clone(self, new_id, inputs):
        return replace(self, id=new_id, inputs=list(inputs), copy_of=self.id if self.copy_of < 0 else self.copy_of)


@dataclass
class Graph:
    """The unfused decomposed list L (SSA, execution order); ids == positions."""
    nodes: list
    output: int
    batch: int
    dtype: str
    orig_flops: dict = field(default_factory=dict)   # original conv layer -> FLOPs (R1 threshold)
    nodes_by_id: dict = field(default_factory=dict)  # every node ever created (L and COPY clones)

    def size(self, v: Node) -> int:
        return self.batch * v.C * v.H * v.W * DTYPE_BYTES[self.dtype]


def _out_hw(h, w, kh, kw, sh, sw, ph, pw):
    return (h + 2 * ph - kh) // sh + 1, (w + 2 * pw - kw) // sw + 1


def expand(model) -> Graph:
    """O1: expand each decomposed conv of the original layer graph into its
    role-tagged sequence; all other layers are kept as they are.  Returns the
    unfused decomposed list L (the paper's "Decomposed" baseline)."""
    nodes: list = []
    out_of: dict = {}
    orig_flops: dict = {}

    def push(**kw):
        n = Node(id=len(nodes), **kw)
        nodes.append(n)
        return n

    for li, layer in enumerate(model.layers):
        ins = [out_of[i] for i in layer.inputs]
        src = [nodes[i] for i in ins]
        if layer.op == "input":
            n = push(op="input", inputs=[], orig=li, name=layer.name,
                     C=model.channels, H=model.height, W=model.width)
        elif layer.op == "conv":
            x = src[0]
            k, s, p = layer.kernel, layer.stride, layer.pad
            ho, wo = _out_hw(x.H, x.W, k, k, s, s, p, p)
            # FLOPs of the original (undecomposed) conv: COMPUTE_THRESHOLD, P:L219 / R1
            orig_flops[li] = 2 * (x.C // layer.groups) * layer.out_channels * k * k * ho * wo * model.batch
            d = model.decomps.get(li)
            if d is None:
                n = push(op="conv", inputs=ins, orig=li, name=layer.name, kh=k, kw=k, sh=s, sw=s, ph=p, pw=p,
                         groups=layer.groups, C=layer.out_channels, H=ho, W=wo,
                         weight=layer.weight, bias=layer.bias)
            elif d.kind == "tucker2":
                cur = x
                if d.first is not None:                       # fconv: C_in -> R_in
                    cur = push(op="conv", inputs=[cur.id], role="fconv", orig=li, name=layer.name + ".fconv",
                               C=d.rank_in, H=cur.H, W=cur.W, weight=np.asarray(d.first)[:, :, None, None])
                has_last = d.last is not None
                cur = push(op="conv", inputs=[cur.id], role="core", orig=li, name=layer.name + ".core",
                           kh=k, kw=k, sh=s, sw=s, ph=p, pw=p, C=d.rank_out, H=ho, W=wo,
                           weight=np.asarray(d.core), bias=None if has_last else layer.bias)
                if has_last:                                   # lconv: R_out -> C_out
                    cur = push(op="conv", inputs=[cur.id], role="lconv", orig=li, name=layer.name + ".lconv",
                               C=layer.out_channels, H=ho, W=wo,
                               weight=np.asarray(d.last)[:, :, None, None], bias=layer.bias)
                n = cur
            elif d.kind == "cp":
                r = d.rank_in
                f = push(op="conv", inputs=[x.id], role="fconv", orig=li, name=layer.name + ".fconv",
                         C=r, H=x.H, W=x.W, weight=np.asarray(d.first)[:, :, None, None])
                h1, _ = _out_hw(x.H, x.W, k, 1, s, 1, p, 0)
                v = push(op="conv", inputs=[f.id], role="core", orig=li, name=layer.name + ".core_v",
                         kh=k, kw=1, sh=s, sw=1, ph=p, pw=0, groups=r, C=r, H=h1, W=x.W,
                         weight=np.asarray(d.core)[:, None, :, None])
                hz = push(op="conv", inputs=[v.id], role="core", orig=li, name=layer.name + ".core_h",
                          kh=1, kw=k, sh=1, sw=s, ph=0, pw=p, groups=r, C=r, H=ho, W=wo,
                          weight=np.asarray(d.core2)[:, None, None, :])
                n = push(op="conv", inputs=[hz.id], role="lconv", orig=li, name=layer.name + ".lconv",
                         C=layer.out_channels, H=ho, W=wo,
                         weight=np.asarray(d.last)[:, :, None, None], bias=layer.bias)
            elif d.kind == "tt":
                # Tensor-Train (P:L73 [28]; reading R33): the weight W[o, i, a, b] in mode
                # order (C_in, K_h, K_w, C_out) as a train of cores G1 [C_in x r1],
                # G2 [r1 x K x r2], G3 [r2 x K x r3], G4 [r3 x C_out]: fconv 1x1 (C_in -> r1),
                # core K x 1 (r1 -> r2, stride (s, 1), pad (p, 0)), core 1 x K (r2 -> r3,
                # stride (1, s), pad (0, p)), lconv 1x1 (r3 -> C_out, bias)
                # (no fconv when r1 == C_in, as for Tucker-2: a full-rank input mode, R17)
                r1, r2, r3 = d.rank_in, d.rank_mid, d.rank_out
                f = x
                if d.first is not None:
                    f = push(op="conv", inputs=[x.id], role="fconv", orig=li, name=layer.name + ".fconv",
                             C=r1, H=x.H, W=x.W, weight=np.asarray(d.first)[:, :, None, None])
                h1, _ = _out_hw(x.H, x.W, k, 1, s, 1, p, 0)
                v = push(op="conv", inputs=[f.id], role="core", orig=li, name=layer.name + ".core_v",
                         kh=k, kw=1, sh=s, sw=1, ph=p, pw=0, C=r2, H=h1, W=x.W,
                         weight=np.asarray(d.core)[:, :, :, None])
                hz = push(op="conv", inputs=[v.id], role="core", orig=li, name=layer.name + ".core_h",
                          kh=1, kw=k, sh=1, sw=s, ph=0, pw=p, C=r3, H=ho, W=wo,
                          weight=np.asarray(d.core2)[:, :, None, :])
                n = push(op="conv", inputs=[hz.id], role="lconv", orig=li, name=layer.name + ".lconv",
                         C=layer.out_channels, H=ho, W=wo,
                         weight=np.asarray(d.last)[:, :, None, None], bias=layer.bias)
            else:
                raise ValueError(d.kind)
        elif layer.op == "conv_transpose":
            # UNet up-conv, Tucker-2 like a conv (fconv -> core ->
            # lconv); the core is the transposed conv on the reduced channels
            x = src[0]
            k, s, p = layer.kernel, layer.stride, layer.pad
            ho, wo = (x.H - 1) * s - 2 * p + k, (x.W - 1) * s - 2 * p + k
            orig_flops[li] = 2 * x.C * layer.out_channels * k * k * x.H * x.W * model.batch
            d = model.decomps.get(li)
            if d is None:
                n = push(op="convt", inputs=ins, orig=li, name=layer.name, kh=k, kw=k, sh=s, sw=s, ph=p, pw=p,
                         C=layer.out_channels, H=ho, W=wo, weight=layer.weight, bias=layer.bias)
            else:
                assert d.kind == "tucker2"
                cur = x
                if d.first is not None:
                    cur = push(op="conv", inputs=[cur.id], role="fconv", orig=li, name=layer.name + ".fconv",
                               C=d.rank_in, H=cur.H, W=cur.W, weight=np.asarray(d.first)[:, :, None, None])
                has_last = d.last is not None
                cur = push(op="convt", inputs=[cur.id], role="core", orig=li, name=layer.name + ".core",
                           kh=k, kw=k, sh=s, sw=s, ph=p, pw=p, C=d.rank_out, H=ho, W=wo,
                           weight=np.asarray(d.core), bias=None if has_last else layer.bias)
                if has_last:
                    cur = push(op="conv", inputs=[cur.id], role="lconv", orig=li, name=layer.name + ".lconv",
                               C=layer.out_channels, H=ho, W=wo,
                               weight=np.asarray(d.last)[:, :, None, None], bias=layer.bias)
                n = cur
        elif layer.op == "bn":
            x = src[0]
            n = push(op="bn", inputs=ins, orig=li, name=layer.name, C=x.C, H=x.H, W=x.W,
                     bn=(layer.bn_gamma, layer.bn_beta, layer.bn_mean, layer.bn_var, layer.bn_eps))
        elif layer.op in ("relu", "silu"):
            x = src[0]
            n = push(op=layer.op, inputs=ins, orig=li, name=layer.name, C=x.C, H=x.H, W=x.W)
        elif layer.op == "add":
            x = src[0]
            n = push(op="add", inputs=ins, orig=li, name=layer.name, C=x.C, H=x.H, W=x.W)
        elif layer.op == "concat":
            n = push(op="concat", inputs=ins, orig=li, name=layer.name,
                     C=sum(s_.C for s_ in src), H=src[0].H, W=src[0].W)
        elif layer.op == "maxpool":
            x = src[0]
            k, s, p = layer.kernel, layer.stride, layer.pad
            ho, wo = _out_hw(x.H, x.W, k, k, s, s, p, p)
            n = push(op="maxpool", inputs=ins, orig=li, name=layer.name, kh=k, kw=k, sh=s, sw=s, ph=p, pw=p,
                     C=x.C, H=ho, W=wo)
        elif layer.op == "avgpool":
            x = src[0]
            k, s = layer.kernel, layer.stride
            ho, wo = _out_hw(x.H, x.W, k, k, s, s, 0, 0)
            n = push(op="avgpool", inputs=ins, orig=li, name=layer.name, kh=k, kw=k, sh=s, sw=s,
                     C=x.C, H=ho, W=wo)
        elif layer.op == "gap":
            x = src[0]
            n = push(op="gap", inputs=ins, orig=li, name=layer.name, C=x.C, H=1, W=1)
        elif layer.op == "linear":
            n = push(op="linear", inputs=ins, orig=li, name=layer.name, C=layer.out_channels, H=1, W=1,
                     weight=layer.weight, bias=layer.bias)
        else:
            raise ValueError(f"unsupported op {layer.op}")
        out_of[li] = n.id
    return Graph(nodes=nodes, output=out_of[len(model.layers) - 1], batch=model.batch,
                 dtype=model.dtype, orig_flops=orig_flops, nodes_by_id={n.id: n for n in nodes})


def flops(g: Graph, v: Node) -> int:
    """FLOPs of one node of L or O at the graph's batch (reading R1): conv
    2*(C_in/groups)*C_out*kh*kw*H'*W'; transposed conv 2*C_in*C_out*kh*kw*H*W (per input
    pixel); bn 2/elt; relu, add 1/elt (per extra
    input); silu 4/elt; pools kh*kw per output elt; concat 0; gap 1 per input
    elt; linear 2*in*out."""
    N = g.batch
    numel = N * v.C * v.H * v.W
    if v.op == "conv":
        cin = g.nodes_by_id[v.inputs[0]].C
        return 2 * (cin // v.groups) * v.C * v.kh * v.kw * v.H * v.W * N
    if v.op == "convt":
        x = g.nodes_by_id[v.inputs[0]]
        return 2 * x.C * v.C * v.kh * v.kw * x.H * x.W * N
    if v.op == "bn":
        return 2 * numel
    if v.op == "relu":
        return numel
    if v.op == "silu":
        return 4 * numel
    if v.op == "add":
        return (len(v.inputs) - 1) * numel
    if v.op in ("maxpool", "avgpool"):
        return v.kh * v.kw * numel
    if v.op == "gap":
        x = g.nodes_by_id[v.inputs[0]]
        return N * x.C * x.H * x.W
    if v.op == "linear":
        x = g.nodes_by_id[v.inputs[0]]
        return 2 * x.C * x.H * x.W * v.C * N
    return 0
