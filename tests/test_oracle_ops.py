"""Pins for the oracle's fp64 operators (oracle/ops.py).

Each operator is checked against an independent implementation: PyTorch's CPU
reference operators in float64 (a library routine computing the textbook
definition) and, for the convolution, a pure-Python 7-nested loop on tiny
inputs.  A transposed weight, a wrong stride/padding convention or a dropped
bias fails one of these."""
import itertools

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from oracle import ops


def _nchw(x):
    return torch.from_numpy(np.ascontiguousarray(np.transpose(x, (0, 3, 1, 2))))


def _nhwc(t):
    return np.transpose(t.numpy(), (0, 2, 3, 1))


@pytest.mark.parametrize("c,o,k,s,p,groups,kh,kw", [
    (4, 6, 3, 1, 1, 1, 3, 3), (5, 7, 3, 2, 1, 1, 3, 3), (3, 8, 7, 2, 3, 1, 7, 7),
    (6, 6, 3, 1, 1, 6, 3, 1), (6, 6, 3, 2, 1, 6, 1, 3), (8, 4, 1, 1, 0, 1, 1, 1),
    (4, 8, 3, 1, 1, 2, 3, 3), (16, 16, 1, 2, 0, 1, 1, 1),
])
def test_conv2d_matches_torch(c, o, k, s, p, groups, kh, kw):
    rng = np.random.default_rng(0)
    x = rng.standard_normal((2, 9, 11, c))
    w = rng.standard_normal((o, c // groups, kh, kw))
    b = rng.standard_normal(o)
    sh, sw = (s, 1) if kw == 1 and kh > 1 else ((1, s) if kh == 1 and kw > 1 else (s, s))
    ph, pw = (p, 0) if kw == 1 and kh > 1 else ((0, p) if kh == 1 and kw > 1 else (p, p))
    got = ops.conv2d(x, w, b, (sh, sw), (ph, pw), groups)
    ref = F.conv2d(_nchw(x), torch.from_numpy(w), torch.from_numpy(b), stride=(sh, sw), padding=(ph, pw), groups=groups)
    np.testing.assert_allclose(got, _nhwc(ref), rtol=1e-12, atol=1e-12)


def test_conv2d_matches_python_loops():
    """Tiny case against the literal 7-nested loop (no numpy slicing)."""
    rng = np.random.default_rng(1)
    N, H, W, C, O, K, S, P = 1, 5, 4, 3, 2, 3, 2, 1
    x = rng.standard_normal((N, H, W, C))
    w = rng.standard_normal((O, C, K, K))
    got = ops.conv2d(x, w, None, (S, S), (P, P), 1)
    Ho, Wo = (H + 2 * P - K) // S + 1, (W + 2 * P - K) // S + 1
    ref = np.zeros((N, Ho, Wo, O))
    for n, ho, wo, o, i, a, b in itertools.product(range(N), range(Ho), range(Wo), range(O), range(C), range(K), range(K)):
        h, ww = ho * S - P + a, wo * S - P + b
        if 0 <= h < H and 0 <= ww < W:
            ref[n, ho, wo, o] += w[o, i, a, b] * x[n, h, ww, i]
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


def test_pools_bn_linear_match_torch():
    rng = np.random.default_rng(2)
    x = rng.standard_normal((2, 9, 10, 5))
    np.testing.assert_allclose(ops.maxpool(x, 3, 2, 1), _nhwc(F.max_pool2d(_nchw(x), 3, 2, 1)), rtol=0, atol=0)
    np.testing.assert_allclose(ops.maxpool(x, 2, 2, 0), _nhwc(F.max_pool2d(_nchw(x), 2, 2, 0)), rtol=0, atol=0)
    np.testing.assert_allclose(ops.avgpool(x, 2, 2), _nhwc(F.avg_pool2d(_nchw(x), 2, 2)), rtol=1e-14, atol=1e-14)
    np.testing.assert_allclose(ops.gap(x)[:, 0, 0, :], x.mean(axis=(1, 2)), rtol=1e-14)
    g, b, m, v = (rng.uniform(0.5, 1.5, 5), rng.standard_normal(5), rng.standard_normal(5), rng.uniform(0.5, 1.5, 5))
    ref = F.batch_norm(_nchw(x), torch.from_numpy(m), torch.from_numpy(v), torch.from_numpy(g), torch.from_numpy(b),
                       training=False, eps=1e-5)
    np.testing.assert_allclose(ops.batchnorm(x, g, b, m, v, 1e-5), _nhwc(ref), rtol=1e-12, atol=1e-12)
    wl = rng.standard_normal((7, 5 * 9 * 10))
    bl = rng.standard_normal(7)
    ref = F.linear(_nchw(x).reshape(2, -1), torch.from_numpy(wl), torch.from_numpy(bl))
    np.testing.assert_allclose(ops.linear(x, wl, bl)[:, 0, 0, :], ref.numpy(), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(ops.relu(x), np.where(x > 0, x, 0))
    np.testing.assert_allclose(ops.silu(x), _nhwc(F.silu(_nchw(x))), rtol=1e-12, atol=1e-12)


def test_add_and_concat_match_torch_with_channel_order():
    """ops.add is the elementwise sum of all inputs; ops.concat stacks channels in
    input order (Fig. 9 concat split: the first input's channels come first)."""
    rng = np.random.default_rng(3)
    xs = [rng.standard_normal((2, 5, 4, c)) for c in (3, 5, 2)]
    got = ops.concat(xs)
    ref = torch.cat([_nchw(x) for x in xs], dim=1)
    np.testing.assert_array_equal(got, _nhwc(ref))
    # channel order pinned by distinct constants per input
    cs = [np.full((1, 2, 2, c), float(k + 1)) for k, c in enumerate((3, 5, 2))]
    cat = ops.concat(cs)
    assert cat.shape == (1, 2, 2, 10)
    np.testing.assert_array_equal(cat[0, 0, 0], [1, 1, 1, 2, 2, 2, 2, 2, 3, 3])
    same = [rng.standard_normal((2, 5, 4, 6)) for _ in range(3)]
    np.testing.assert_allclose(ops.add(same), _nhwc(torch.stack([_nchw(x) for x in same]).sum(0)), rtol=1e-14)
    np.testing.assert_allclose(ops.add(same[:2]), same[0] + same[1], rtol=0, atol=0)
    # ops.add does not alias or modify its first input
    before = same[0].copy()
    ops.add(same)
    np.testing.assert_array_equal(same[0], before)


@pytest.mark.parametrize("c,o,k,s,p", [(4, 6, 2, 2, 0), (3, 5, 3, 2, 1), (6, 4, 4, 2, 1), (5, 5, 3, 1, 1)])
def test_conv_transpose2d_matches_torch(c, o, k, s, p):
    rng = np.random.default_rng(7)
    x = rng.standard_normal((2, 5, 6, c))
    w = rng.standard_normal((c, o, k, k))
    b = rng.standard_normal(o)
    got = ops.conv_transpose2d(x, w, b, s, p)
    ref = F.conv_transpose2d(_nchw(x), torch.from_numpy(w), torch.from_numpy(b), stride=s, padding=p)
    np.testing.assert_allclose(got, _nhwc(ref), rtol=1e-12, atol=1e-12)


def test_conv_transpose2d_literal_loop():
    """The scatter definition written as plain loops on a tiny input."""
    rng = np.random.default_rng(8)
    x = rng.standard_normal((1, 2, 3, 2))
    w = rng.standard_normal((2, 3, 3, 3))
    s, p = 2, 1
    got = ops.conv_transpose2d(x, w, None, s, p)
    ho, wo = (2 - 1) * s - 2 * p + 3, (3 - 1) * s - 2 * p + 3
    ref = np.zeros((1, ho, wo, 3))
    for ih, iw, ci, oc, i, j in itertools.product(range(2), range(3), range(2), range(3), range(3), range(3)):
        oh, ow = ih * s - p + i, iw * s - p + j
        if 0 <= oh < ho and 0 <= ow < wo:
            ref[0, oh, ow, oc] += x[0, ih, iw, ci] * w[ci, oc, i, j]
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)
