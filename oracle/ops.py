"""fp64 reference operators (oracle; test infrastructure only).

Tensors are NHWC float64 numpy arrays [N, H, W, C].  Every operator is the
textbook definition written as directly as numpy allows: the convolution is
the sum over kernel taps (kh, kw) of a channel contraction of the shifted,
zero-padded input -- i.e. the 7-nested direct loop with the batch / spatial /
channel loops handed to numpy.  No blocking, fusion or reordering.

The paper uses the standard CNN operators of its
PyTorch models; their definitions (cross-correlation with zero padding, BN in
inference form, max pooling with -inf padding, average pooling, global average
pooling, linear over the NCHW-flattened features) are taken as the plain
semantics (SURVEY.md 8(c) "What is the result").
"""
from __future__ import annotations

import numpy as np


def conv2d(x, w, bias, stride, pad, groups):
    """out[n,ho,wo,o] = bias[o] + sum_{i,kh,kw} w[o,i,kh,kw] *
    xpad[n, ho*sh+kh, wo*sw+kw, g(o)*Cg + i]   (cross-correlation).

    x [N,H,W,C]; w [O, C/groups, KH, KW] (PyTorch OIHW); stride/pad (h, w)."""
    n, h, wd, c = x.shape
    o, cg, kh, kw = w.shape
    sh, sw = stride
    ph, pw = pad
    assert c == cg * groups and o % groups == 0
    og = o // groups
    ho = (h + 2 * ph - kh) // sh + 1
    wo = (wd + 2 * pw - kw) // sw + 1
    xp = np.zeros((n, h + 2 * ph, wd + 2 * pw, c), np.float64)
    xp[:, ph:ph + h, pw:pw + wd, :] = x
    out = np.zeros((n, ho, wo, o), np.float64)
    w = np.asarray(w, np.float64)
    for i in range(kh):
        for j in range(kw):
            tap = xp[:, i:i + sh * (ho - 1) + 1:sh, j:j + sw * (wo - 1) + 1:sw, :]
            if groups == 1:
                out += tap @ w[:, :, i, j].T
            elif cg == 1 and og == 1:          # depthwise: one input channel per output
                out += tap * w[:, 0, i, j]
            else:
                for g in range(groups):
                    out[..., g * og:(g + 1) * og] += tap[..., g * cg:(g + 1) * cg] @ w[g * og:(g + 1) * og, :, i, j].T
    if bias is not None:
        out += np.asarray(bias, np.float64)
    return out


def conv_transpose2d(x, w, bias, stride, pad):
    """Transposed convolution (UNet up-conv): every input pixel scatters through every
    tap, out[n, ih*s + i - p, iw*s + j - p, o] += sum_c x[n, ih, iw, c] * w[c, o, i, j]
    (w in PyTorch ConvTranspose2d layout [C_in, C_out, kh, kw]); then the p-border is
    cropped.  Output size (H - 1) * s - 2p + k."""
    n, h, wd, c = x.shape
    ci, o, kh, kw = w.shape
    assert ci == c
    s, p = stride, pad
    full = np.zeros((n, (h - 1) * s + kh, (wd - 1) * s + kw, o), np.float64)
    w = np.asarray(w, np.float64)
    for i in range(kh):
        for j in range(kw):
            full[:, i:i + s * (h - 1) + 1:s, j:j + s * (wd - 1) + 1:s, :] += x @ w[:, :, i, j]
    out = full[:, p:full.shape[1] - p, p:full.shape[2] - p, :]
    if bias is not None:
        out = out + np.asarray(bias, np.float64)
    return np.ascontiguousarray(out)


def batchnorm(x, gamma, beta, mean, var, eps):
    """y = gamma * (x - mean) / sqrt(var + eps) + beta, per channel."""
    g = np.asarray(gamma, np.float64)
    return g * (x - np.asarray(mean, np.float64)) / np.sqrt(np.asarray(var, np.float64) + eps) + np.asarray(beta, np.float64)


def relu(x):
    return np.maximum(x, 0.0)


def silu(x):
    return x / (1.0 + np.exp(-x))


def add(xs):
    out = np.array(xs[0], np.float64, copy=True)
    for t in xs[1:]:
        out = out + t
    return out


def concat(xs):
    return np.concatenate(xs, axis=3)


def maxpool(x, k, s, p):
    """max over the k x k window with stride s, padding p filled with -inf."""
    n, h, w, c = x.shape
    ho = (h + 2 * p - k) // s + 1
    wo = (w + 2 * p - k) // s + 1
    xp = np.full((n, h + 2 * p, w + 2 * p, c), -np.inf)
    xp[:, p:p + h, p:p + w, :] = x
    out = np.full((n, ho, wo, c), -np.inf)
    for i in range(k):
        for j in range(k):
            out = np.maximum(out, xp[:, i:i + s * (ho - 1) + 1:s, j:j + s * (wo - 1) + 1:s, :])
    return out


def avgpool(x, k, s):
    """mean over the k x k window with stride s, no padding."""
    n, h, w, c = x.shape
    ho = (h - k) // s + 1
    wo = (w - k) // s + 1
    out = np.zeros((n, ho, wo, c), np.float64)
    for i in range(k):
        for j in range(k):
            out += x[:, i:i + s * (ho - 1) + 1:s, j:j + s * (wo - 1) + 1:s, :]
    return out / (k * k)


def gap(x):
    """global average pool -> [N, 1, 1, C]."""
    return x.mean(axis=(1, 2), keepdims=True)


def linear(x, w, b):
    """y = flatten_NCHW(x) @ w.T + b; flatten order is c-major (torchvision)."""
    n = x.shape[0]
    flat = np.transpose(x, (0, 3, 1, 2)).reshape(n, -1)
    y = flat @ np.asarray(w, np.float64).T
    if b is not None:
        y = y + np.asarray(b, np.float64)
    return y.reshape(n, 1, 1, -1)
