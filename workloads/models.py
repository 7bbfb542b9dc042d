"""Seeded builders for the original (undecomposed) layer graphs and their
decomposition factors.

Everything here is *input*: the shapes follow the paper's workloads (ResNet,
VGG, DenseNet on ILSVRC-sized 224x224 RGB images) and the
configs of BASELINE.json; the values are random (there are no datasets or
trained weights).  The recipe is stated in DESIGN.md section "Input recipe".

Graph format (consumed independently by `oracle/` and by the C ABI binding):
  * `Model.layers` is an SSA list in execution order; `layers[0]` is the input.
    `Layer.inputs` holds indices of earlier layers.  The last layer is the
    graph output.
  * `Model.decomps[i]` gives the decomposition factors of conv layer i:
      Tucker-2 : first [R_in, C_in] (None iff R_in == C_in),
                 core  [R_out, R_in, K, K],
                 last  [C_out, R_out] (None iff R_out == C_out)
      CP       : first [R, C_in], core = Kv [R, K], core2 = Kh [R, K],
                 last [C_out, R]
  * Tensors are NHWC at the boundary; weights follow PyTorch conventions
    (conv OIHW, linear [out, in] with `in` flattened in NCHW c-major order).
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Optional

import numpy as np

F32 = "f32"
BF16 = "bf16"


def rank_rule(c: int) -> int:
    """Decomposition rank for a mode of size c: 8*ceil(0.1*c/8).

    PAPER.md P:L345 fixes only the "decomposition ratio of 0.1"; the rounding
    to a multiple of 8 is reading R15 so that bf16 rows of the
    reduced tensors are 16-byte aligned.  Integer arithmetic: ceil(c/80)*8.
    """
    return 8 * ((c + 79) // 80)


def bf16_round(x: np.ndarray) -> np.ndarray:
    """Round float32 values to the nearest bfloat16 (ties to even), returned as
    float32.  Used so that bf16 workloads hand the oracle and the GPU path the
    very same representable values."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    u = x.view(np.uint32).astype(np.uint64)
    rounding = ((u >> 16) & 1) + 0x7FFF
    u = ((u + rounding) & 0xFFFF0000).astype(np.uint32)
    return u.view(np.float32).reshape(x.shape)


@dataclass
class Layer:
    op: str                      # input conv bn relu silu add concat maxpool avgpool gap linear
    inputs: list
    name: str = ""
    out_channels: int = 0        # conv / linear / input
    kernel: int = 1              # conv / pool
    stride: int = 1
    pad: int = 0
    groups: int = 1
    weight: Optional[np.ndarray] = None   # conv OIHW (may be None when decomposed), linear [out, in]
    bias: Optional[np.ndarray] = None
    bn_gamma: Optional[np.ndarray] = None
    bn_beta: Optional[np.ndarray] = None
    bn_mean: Optional[np.ndarray] = None
    bn_var: Optional[np.ndarray] = None
    bn_eps: float = 1e-5


@dataclass
class Decomp:
    layer: int
    kind: str                    # "tucker2" | "cp" | "tt"
    rank_in: int
    rank_out: int
    first: Optional[np.ndarray]
    core: np.ndarray
    core2: Optional[np.ndarray]
    last: Optional[np.ndarray]
    rank_mid: int = 0            # Tensor-Train: the rank between the two cores


@dataclass
class Model:
    name: str
    batch: int
    height: int
    width: int
    channels: int
    dtype: str
    layers: list = field(default_factory=list)
    decomps: dict = field(default_factory=dict)
    input_seed: int = 1234

    @property
    def output(self) -> int:
        return len(self.layers) - 1


def skip_edges(model: Model) -> list:
    """All (src, dst) input edges with dst - src > 1 in layer order: the skip
    edges the C ABI expects ("Skip-edge validation")."""
    edges = []
    for dst, l in enumerate(model.layers):
        for src in l.inputs:
            if dst - src > 1:
                edges.append((src, dst))
    return edges


def make_input(model: Model, start: int = 0, count: Optional[int] = None) -> np.ndarray:
    """Images [count, H, W, C] float32 (NHWC), image i drawn from its own
    generator seeded by input_seed + i, so any shard equals the same images of
    a single-GPU batch."""
    if count is None:
        count = model.batch
    out = np.empty((count, model.height, model.width, model.channels), np.float32)
    for k in range(count):
        rng = np.random.default_rng(model.input_seed + start + k)
        out[k] = rng.standard_normal((model.height, model.width, model.channels), dtype=np.float32)
    if model.dtype == BF16:
        out = bf16_round(out)
    return out


# ----------------------------------------------------------------------------
# builder helpers
# ----------------------------------------------------------------------------

class _G:
    """Appends layers, tracks (C, H, W) per layer, draws seeded weights."""

    def __init__(self, name, batch, h, w, c, dtype, seed, rank=rank_rule, cp=False, tt=False):
        self.m = Model(name, batch, h, w, c, dtype)
        self.m.layers.append(Layer("input", [], name="input", out_channels=c))
        self.shape = [(c, h, w)]
        self.seed = seed
        self.rank = rank
        self.cp = cp
        self.tt = tt

    def rng(self):
        return np.random.default_rng(self.seed * 1_000_003 + len(self.m.layers))

    def _q(self, x):
        return bf16_round(x) if self.m.dtype == BF16 else np.asarray(x, np.float32)

    def _add(self, layer, shape):
        self.m.layers.append(layer)
        self.shape.append(shape)
        return len(self.m.layers) - 1

    @staticmethod
    def _orth(rng, rows, cols):
        """rows x cols with orthonormal columns (rows >= cols) via QR."""
        a = rng.standard_normal((rows, cols))
        q, r = np.linalg.qr(a)
        q = q * np.sign(np.diag(r))[None, :]
        return q

    def conv(self, x, cout, k, s=1, p=0, bias=False, name="", ranks=None):
        cin, h, w = self.shape[x]
        rng = self.rng()
        idx = len(self.m.layers)
        b = self._q(rng.normal(0.0, 0.01, cout).astype(np.float32)) if bias else None
        layer = Layer("conv", [x], name=name, out_channels=cout, kernel=k, stride=s, pad=p, bias=b)
        if self.cp:
            r = self.rank(cout) if ranks is None else ranks[0]
            if r <= cin:
                first = self._orth(rng, cin, r).T
            else:
                first = rng.standard_normal((r, cin)) / np.sqrt(cin)
            kv = rng.standard_normal((r, k)) / np.sqrt(k)
            kh = rng.standard_normal((r, k)) / np.sqrt(k)
            last = rng.standard_normal((cout, r)) * np.sqrt(2.0 / r)
            d = Decomp(idx, "cp", r, r, self._q(first), self._q(kv), self._q(kh), self._q(last))
        elif self.tt and k > 1:
            # Tensor-Train (reading R33): r1 = R(C_in), r2 = r3 = R(C_out); orthonormal outer
            # factors as for Tucker-2, Gaussian cores scaled by their fan-in
            r1 = min(self.rank(cin), cin) if ranks is None else ranks[0]
            r3 = min(self.rank(cout), cout) if ranks is None else ranks[1]
            r2 = r3
            first = self._orth(rng, cin, r1).T if r1 < cin else None       # no fconv on a full-rank mode
            cv = rng.standard_normal((r2, r1, k)) / np.sqrt(r1 * k)
            ch = rng.standard_normal((r3, r2, k)) / np.sqrt(r2 * k)
            last = self._orth(rng, cout, r3) * np.sqrt(cout / r3) if r3 <= cout else \
                rng.standard_normal((cout, r3)) * np.sqrt(2.0 / r3)
            d = Decomp(idx, "tt", r1, r3, None if first is None else self._q(first), self._q(cv), self._q(ch),
                       self._q(last), rank_mid=r2)
        else:
            ri = self.rank(cin) if ranks is None else ranks[0]
            ro = self.rank(cout) if ranks is None else ranks[1]
            ri, ro = min(ri, cin), min(ro, cout)
            first = self._orth(rng, cin, ri).T if ri < cin else None
            core = rng.standard_normal((ro, ri, k, k)) / np.sqrt(ri * k * k)
            last = self._orth(rng, cout, ro) * np.sqrt(cout / ro) if ro < cout else None
            d = Decomp(idx, "tucker2", ri, ro,
                       None if first is None else self._q(first), self._q(core), None,
                       None if last is None else self._q(last))
        self.m.decomps[idx] = d
        ho = (h + 2 * p - k) // s + 1
        wo = (w + 2 * p - k) // s + 1
        return self._add(layer, (cout, ho, wo))

    def conv_transpose(self, x, cout, k, s, p=0, bias=False, name=""):
        """ConvTranspose2d (UNet up-conv), Tucker-2 decomposed with R(c): first [R_in, C_in],
        core [R_in, R_out, k, k] (transposed-conv layout), last [C_out, R_out]."""
        cin, h, w = self.shape[x]
        rng = self.rng()
        idx = len(self.m.layers)
        b = self._q(rng.normal(0.0, 0.01, cout).astype(np.float32)) if bias else None
        layer = Layer("conv_transpose", [x], name=name, out_channels=cout, kernel=k, stride=s, pad=p, bias=b)
        ri, ro = min(self.rank(cin), cin), min(self.rank(cout), cout)
        first = self._orth(rng, cin, ri).T if ri < cin else None
        # each output pixel meets ~ (k/s)^2 taps of R_in channels
        core = rng.standard_normal((ri, ro, k, k)) / np.sqrt(ri * max(1.0, (k / s) ** 2))
        last = self._orth(rng, cout, ro) * np.sqrt(cout / ro) if ro < cout else None
        self.m.decomps[idx] = Decomp(idx, "tucker2", ri, ro, None if first is None else self._q(first),
                                     self._q(core), None, None if last is None else self._q(last))
        return self._add(layer, (cout, (h - 1) * s - 2 * p + k, (w - 1) * s - 2 * p + k))

    def bn(self, x, name=""):
        c, h, w = self.shape[x]
        rng = self.rng()
        layer = Layer("bn", [x], name=name,
                      bn_gamma=rng.uniform(0.8, 1.2, c).astype(np.float32),
                      bn_beta=rng.normal(0.0, 0.05, c).astype(np.float32),
                      bn_mean=rng.normal(0.0, 0.05, c).astype(np.float32),
                      bn_var=rng.uniform(0.8, 1.2, c).astype(np.float32))
        return self._add(layer, (c, h, w))

    def relu(self, x, name=""):
        return self._add(Layer("relu", [x], name=name), self.shape[x])

    def add(self, xs, name=""):
        return self._add(Layer("add", list(xs), name=name), self.shape[xs[0]])

    def concat(self, xs, name=""):
        c = sum(self.shape[x][0] for x in xs)
        _, h, w = self.shape[xs[0]]
        return self._add(Layer("concat", list(xs), name=name), (c, h, w))

    def maxpool(self, x, k, s, p=0, name=""):
        c, h, w = self.shape[x]
        return self._add(Layer("maxpool", [x], name=name, kernel=k, stride=s, pad=p),
                         (c, (h + 2 * p - k) // s + 1, (w + 2 * p - k) // s + 1))

    def avgpool(self, x, k, s, name=""):
        c, h, w = self.shape[x]
        return self._add(Layer("avgpool", [x], name=name, kernel=k, stride=s),
                         (c, (h - k) // s + 1, (w - k) // s + 1))

    def gap(self, x, name=""):
        c, _, _ = self.shape[x]
        return self._add(Layer("gap", [x], name=name), (c, 1, 1))

    def linear(self, x, out, name="", gain=1.0):
        c, h, w = self.shape[x]
        fan_in = c * h * w
        rng = self.rng()
        wgt = rng.standard_normal((out, fan_in), dtype=np.float32) * np.float32(np.sqrt(gain / fan_in))
        b = rng.normal(0.0, 0.01, out).astype(np.float32)
        return self._add(Layer("linear", [x], name=name, out_channels=out,
                               weight=self._q(wgt), bias=self._q(b)), (out, 1, 1))


# ----------------------------------------------------------------------------
# configs
# ----------------------------------------------------------------------------

def c1_basic_block(dtype=F32, batch=1, seed=11):
    """BASELINE.json configs[0]: one Tucker-2 ResNet basic block, input
    1x16x8x8, ranks 4/4, fp32; the identity skip is the graph input."""
    g = _G("c1_basic_block", batch, 8, 8, 16, dtype, seed, rank=lambda c: 4)
    x = 0
    a = g.relu(g.bn(g.conv(x, 16, 3, 1, 1, name="conv1"), "bn1"), "relu1")
    b = g.bn(g.conv(a, 16, 3, 1, 1, name="conv2"), "bn2")
    g.relu(g.add([b, x], "add"), "relu2")
    return g.m


def t1_chain(dtype=F32, batch=1, seed=21):
    """Fig. 3b chain: tk(64->64, 8, 8) -> ReLU -> tk."""
    g = _G("t1_chain", batch, 8, 8, 64, dtype, seed, rank=lambda c: 8)
    a = g.relu(g.conv(0, 64, 3, 1, 1, name="conv1"), "relu")
    g.conv(a, 64, 3, 1, 1, name="conv2")
    return g.m


def t2_stem_blocks(n_blocks=1, dtype=F32, batch=1, seed=31):
    """Fig. 7/8 style: decomposed stem 3->16 then n basic blocks (16 ch, rank 4)."""
    g = _G(f"t2_stem_{n_blocks}blocks", batch, 8, 8, 3, dtype, seed, rank=lambda c: min(c, 4))
    x = g.relu(g.bn(g.conv(0, 16, 3, 1, 1, name="stem"), "stem.bn"), "stem.relu")
    for i in range(n_blocks):
        a = g.relu(g.bn(g.conv(x, 16, 3, 1, 1, name=f"b{i}.conv1"), f"b{i}.bn1"), f"b{i}.relu1")
        b = g.bn(g.conv(a, 16, 3, 1, 1, name=f"b{i}.conv2"), f"b{i}.bn2")
        x = g.relu(g.add([b, x], f"b{i}.add"), f"b{i}.relu2")
    return g.m


def t3_mini_bottleneck(dtype=F32, batch=1, seed=41):
    """Mini ResNet-50: stem 7x7 s1 + maxpool, two bottlenecks (mid 8, out 32),
    downsample evaluated after conv3 (torchvision order, reading R24)."""
    g = _G("t3_mini_bottleneck", batch, 16, 16, 3, dtype, seed)

    def tk(x, cout, ri, ro, k, s=1, p=0, name=""):
        return g.conv(x, cout, k, s, p, name=name, ranks=(ri, ro))

    x = g.maxpool(g.relu(g.bn(tk(0, 8, 3, 2, 7, 1, 3, "stem"), "stem.bn"), "stem.relu"), 3, 2, 1, "stem.pool")
    for i in range(2):
        cin = g.shape[x][0]
        a = g.relu(g.bn(tk(x, 8, 2, 2, 1, name=f"b{i}.conv1"), f"b{i}.bn1"), f"b{i}.relu1")
        b = g.relu(g.bn(tk(a, 8, 2, 2, 3, 1, 1, f"b{i}.conv2"), f"b{i}.bn2"), f"b{i}.relu2")
        c = g.bn(tk(b, 32, 2, 4, 1, name=f"b{i}.conv3"), f"b{i}.bn3")
        sc = x
        if cin != 32:
            sc = g.bn(tk(x, 32, 2, 4, 1, name=f"b{i}.ds"), f"b{i}.ds.bn")
        x = g.relu(g.add([c, sc], f"b{i}.add"), f"b{i}.relu3")
    return g.m


def t4_mini_densenet(dtype=F32, batch=1, seed=51):
    """Mini DenseNet: stem 16 ch, 3 dense layers (growth 8), transition to 20,
    GAP as the graph output."""
    g = _G("t4_mini_densenet", batch, 16, 16, 3, dtype, seed)

    def tk(x, cout, ri, ro, k, s=1, p=0, name=""):
        return g.conv(x, cout, k, s, p, name=name, ranks=(ri, ro))

    stem = g.maxpool(g.relu(g.bn(tk(0, 16, 3, 2, 7, 1, 3, "stem"), "stem.bn"), "stem.relu"), 3, 2, 1, "stem.pool")
    feats = [stem]
    for i in range(3):
        x = feats[0] if len(feats) == 1 else g.concat(feats, f"l{i}.cat")
        a = g.relu(g.bn(x, f"l{i}.bn1"), f"l{i}.relu1")
        a = g.relu(g.bn(tk(a, 32, 2, 2, 1, name=f"l{i}.conv1"), f"l{i}.bn2"), f"l{i}.relu2")
        feats.append(tk(a, 8, 2, 2, 3, 1, 1, f"l{i}.conv2"))
    x = g.concat(feats, "t.cat")
    x = g.relu(g.bn(x, "t.bn"), "t.relu")
    x = g.avgpool(tk(x, 20, 2, 2, 1, name="t.conv"), 2, 2, "t.pool")
    g.gap(x, "gap")
    return g.m


def _basic_block(g, x, cout, stride, name):
    cin = g.shape[x][0]
    a = g.relu(g.bn(g.conv(x, cout, 3, stride, 1, name=f"{name}.conv1"), f"{name}.bn1"), f"{name}.relu1")
    b = g.bn(g.conv(a, cout, 3, 1, 1, name=f"{name}.conv2"), f"{name}.bn2")
    sc = x
    if stride != 1 or cin != cout:
        sc = g.bn(g.conv(x, cout, 1, stride, 0, name=f"{name}.shortcut"), f"{name}.shortcut.bn")
    return g.relu(g.add([b, sc], f"{name}.add"), f"{name}.relu2")


def resnet18_cifar(batch=128, dtype=BF16, height=32, width=32, seed=101, tt=False):
    """BASELINE.json configs[1]: ResNet-18, CIFAR-10 shape (kuangliu layout,
    reading R23): 3x3 s1 stem, no maxpool, widths 64-512, 10 classes.  tt=True: every
    K x K conv Tensor-Train decomposed (reading R33), the 1x1
    shortcut convs Tucker-2."""
    g = _G("resnet18_tt" if tt else "resnet18_cifar", batch, height, width, 3, dtype, seed, tt=tt)
    x = g.relu(g.bn(g.conv(0, 64, 3, 1, 1, name="conv1"), "bn1"), "relu")
    for si, (c, s) in enumerate([(64, 1), (128, 2), (256, 2), (512, 2)]):
        for bi in range(2):
            x = _basic_block(g, x, c, s if bi == 0 else 1, f"layer{si + 1}.{bi}")
    x = g.gap(x, "avgpool")
    g.linear(x, 10, "linear")
    return g.m


def resnet50(batch=256, dtype=BF16, height=224, width=224, seed=202):
    """BASELINE.json configs[2]: ResNet-50 (torchvision v1.5: stride on the
    3x3 conv; downsample evaluated after conv3/bn3, reading R24)."""
    g = _G("resnet50", batch, height, width, 3, dtype, seed)
    x = g.relu(g.bn(g.conv(0, 64, 7, 2, 3, name="conv1"), "bn1"), "relu")
    x = g.maxpool(x, 3, 2, 1, "maxpool")
    for si, (mid, nb, s) in enumerate([(64, 3, 1), (128, 4, 2), (256, 6, 2), (512, 3, 2)]):
        for bi in range(nb):
            name = f"layer{si + 1}.{bi}"
            stride = s if bi == 0 else 1
            cin = g.shape[x][0]
            a = g.relu(g.bn(g.conv(x, mid, 1, name=f"{name}.conv1"), f"{name}.bn1"), f"{name}.relu1")
            b = g.relu(g.bn(g.conv(a, mid, 3, stride, 1, name=f"{name}.conv2"), f"{name}.bn2"), f"{name}.relu2")
            c = g.bn(g.conv(b, mid * 4, 1, name=f"{name}.conv3"), f"{name}.bn3")
            sc = x
            if bi == 0:
                sc = g.bn(g.conv(x, mid * 4, 1, stride, 0, name=f"{name}.downsample.0"), f"{name}.downsample.1")
            x = g.relu(g.add([c, sc], f"{name}.add"), f"{name}.relu3")
    x = g.gap(x, "avgpool")
    g.linear(x, 1000, "fc")
    return g.m


def vgg16_cp(batch=256, dtype=BF16, height=224, width=224, seed=303):
    """BASELINE.json configs[3]: VGG-16 (no BN), every conv CP-decomposed with
    rank R(C_out) (reading R16/R15); classifier 25088-4096-4096-1000 (dropout
    is the identity at inference)."""
    g = _G("vgg16_cp", batch, height, width, 3, dtype, seed, cp=True)
    x = 0
    cfg = [64, 64, "M", 128, 128, "M", 256, 256, 256, "M", 512, 512, 512, "M", 512, 512, 512, "M"]
    ci = 0
    for v in cfg:
        if v == "M":
            x = g.maxpool(x, 2, 2, 0, f"pool{ci}")
        else:
            ci += 1
            x = g.relu(g.conv(x, v, 3, 1, 1, bias=True, name=f"conv{ci}"), f"relu{ci}")
    x = g.relu(g.linear(x, 4096, "fc1", gain=2.0), "fc1.relu")
    x = g.relu(g.linear(x, 4096, "fc2", gain=2.0), "fc2.relu")
    g.linear(x, 1000, "fc3")
    return g.m


def densenet121(batch=128, dtype=BF16, height=224, width=224, seed=404):
    """BASELINE.json configs[4]: DenseNet-121 (growth 32, bn_size 4, blocks
    6-12-24-16, torchvision layout, concat per layer: reading R24)."""
    g = _G("densenet121", batch, height, width, 3, dtype, seed)
    x = g.relu(g.bn(g.conv(0, 64, 7, 2, 3, name="conv0"), "norm0"), "relu0")
    x = g.maxpool(x, 3, 2, 1, "pool0")
    for bi, nl in enumerate([6, 12, 24, 16]):
        feats = [x]
        for li in range(nl):
            name = f"denseblock{bi + 1}.denselayer{li + 1}"
            h = feats[0] if len(feats) == 1 else g.concat(feats, f"{name}.cat")
            h = g.relu(g.bn(h, f"{name}.norm1"), f"{name}.relu1")
            h = g.relu(g.bn(g.conv(h, 128, 1, name=f"{name}.conv1"), f"{name}.norm2"), f"{name}.relu2")
            feats.append(g.conv(h, 32, 3, 1, 1, name=f"{name}.conv2"))
        x = g.concat(feats, f"denseblock{bi + 1}.cat")
        if bi < 3:
            c = g.shape[x][0]
            name = f"transition{bi + 1}"
            x = g.relu(g.bn(x, f"{name}.norm"), f"{name}.relu")
            x = g.avgpool(g.conv(x, c // 2, 1, name=f"{name}.conv"), 2, 2, f"{name}.pool")
    x = g.relu(g.bn(x, "norm5"), "relu5")
    x = g.gap(x, "avgpool")
    g.linear(x, 1000, "classifier")
    return g.m


def alexnet(batch=256, dtype=BF16, height=224, width=224, seed=505):
    """AlexNet (torchvision layout: 5 convs with bias, ReLU, three 3x3/s2 max pools,
    classifier 9216-4096-4096-1000; dropout is the identity at inference), every conv
    Tucker-2 decomposed with R(c) (the paper applies Tucker decomposition to all
    models).  No skip connections: TeMCO applies activation-layer fusion only (P:L345,
    P:L355).  At 224x224 the last pool is 6x6, so torchvision's adaptive average pool
    is the identity and is omitted."""
    g = _G("alexnet", batch, height, width, 3, dtype, seed)
    x = g.relu(g.conv(0, 64, 11, 4, 2, bias=True, name="features.0"), "features.1")
    x = g.maxpool(x, 3, 2, 0, "features.2")
    x = g.relu(g.conv(x, 192, 5, 1, 2, bias=True, name="features.3"), "features.4")
    x = g.maxpool(x, 3, 2, 0, "features.5")
    x = g.relu(g.conv(x, 384, 3, 1, 1, bias=True, name="features.6"), "features.7")
    x = g.relu(g.conv(x, 256, 3, 1, 1, bias=True, name="features.8"), "features.9")
    x = g.relu(g.conv(x, 256, 3, 1, 1, bias=True, name="features.10"), "features.11")
    x = g.maxpool(x, 3, 2, 0, "features.12")
    x = g.relu(g.linear(x, 4096, "classifier.1", gain=2.0), "classifier.2")
    x = g.relu(g.linear(x, 4096, "classifier.4", gain=2.0), "classifier.5")
    g.linear(x, 1000, "classifier.6")
    return g.m


def unet(batch=16, dtype=BF16, height=256, width=256, seed=606, base=64, n_classes=2):
    """UNet (Ronneberger et al. [34], the paper's segmentation model, P:L126 / P:L345 / P:L355):
    four down blocks (2x2 max pool + DoubleConv), four up blocks (2x2 / stride-2 transposed
    conv "up-conv" + channel concat with the encoder feature of the same resolution +
    DoubleConv), DoubleConv = (3x3 conv (no bias) -> BN -> ReLU) x 2, 1x1 output conv to
    n_classes (Carvana masks).  Every conv and up-conv Tucker-2 decomposed with R(c).  The
    encoder features x1..x4 are the long-range skips (76.2 % of the decomposed model's peak
    in the paper's Fig. 4a).  Shape only: the paper's Carvana images are matched in shape."""
    g = _G("unet", batch, height, width, 3, dtype, seed)

    def dconv(x, c, name):
        x = g.relu(g.bn(g.conv(x, c, 3, 1, 1, name=f"{name}.conv1"), f"{name}.bn1"), f"{name}.relu1")
        return g.relu(g.bn(g.conv(x, c, 3, 1, 1, name=f"{name}.conv2"), f"{name}.bn2"), f"{name}.relu2")

    c = [base, base * 2, base * 4, base * 8, base * 16]
    xs = [dconv(0, c[0], "inc")]
    for i in range(1, 5):
        xs.append(dconv(g.maxpool(xs[-1], 2, 2, 0, f"down{i}.pool"), c[i], f"down{i}"))
    x = xs[4]
    for i in range(3, -1, -1):
        u = g.conv_transpose(x, c[i], 2, 2, 0, bias=True, name=f"up{4 - i}.upconv")
        x = dconv(g.concat([xs[i], u], f"up{4 - i}.cat"), c[i], f"up{4 - i}")
    g.conv(x, n_classes, 1, 1, 0, bias=True, name="outc")
    return g.m


CONFIGS = {
    "c1": lambda **kw: c1_basic_block(**kw),
    "resnet18_cifar": lambda **kw: resnet18_cifar(**kw),
    "resnet18_tt": lambda **kw: resnet18_cifar(tt=True, **kw),
    "resnet50": lambda **kw: resnet50(**kw),
    "vgg16_cp": lambda **kw: vgg16_cp(**kw),
    "densenet121": lambda **kw: densenet121(**kw),
    "alexnet": lambda **kw: alexnet(**kw),
    "unet": lambda **kw: unet(**kw),
}


def build_config(name: str, **kw) -> Model:
    return CONFIGS[name](**kw)
