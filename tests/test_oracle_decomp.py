"""Pins for decomposition expansion (oracle step O1, Eq. (2)).

With full ranks the decomposed convolution sequence must reproduce the
original convolution exactly (to fp64 rounding):
  * Tucker-2: orthogonal factor matrices U (C_out x C_out),
    V (C_in x C_in) and core G = U^T x_0 W x_1 V give fconv = V^T, core = G,
    lconv = U, and W = G x_0 U x_1 V.
  * CP (reading R16): rank R = C_in*K^2 with unit-vector factors
    B[(i,a,b), i'] = d(i,i'), Kv[(i,a,b), a'] = d(a,a'), Kh[(i,a,b), b'] = d(b,b'),
    A[o, (i,a,b)] = W[o,i,a,b] reproduces W, including stride and padding.
The reference output is torch's conv2d of the original W (independent library).
"""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import oracle
from workloads import Decomp, Layer, Model


def _single_conv_model(cin, cout, k, s, p, decomp_fn, bias=True, h=9, w=8):
    rng = np.random.default_rng(7)
    W = rng.standard_normal((cout, cin, k, k))
    b = rng.standard_normal(cout) if bias else None
    m = Model("single", 2, h, w, cin, "f32")
    m.layers = [Layer("input", [], out_channels=cin),
                Layer("conv", [0], out_channels=cout, kernel=k, stride=s, pad=p, weight=W, bias=b)]
    m.decomps = {1: decomp_fn(W, rng)}
    return m, W, b


def _ref(m, W, b, x):
    t = F.conv2d(torch.from_numpy(np.transpose(x, (0, 3, 1, 2)).astype(np.float64)), torch.from_numpy(W),
                 None if b is None else torch.from_numpy(b), stride=m.layers[1].stride, padding=m.layers[1].pad)
    return np.transpose(t.numpy(), (0, 2, 3, 1))


def _orth(rng, n):
    q, _ = np.linalg.qr(rng.standard_normal((n, n)))
    return q


def tucker_full(W, rng):
    cout, cin = W.shape[:2]
    U, V = _orth(rng, cout), _orth(rng, cin)
    G = np.einsum("oa,oikl,ib->abkl", U, W, V)
    return Decomp(1, "tucker2", cin, cout, V.T.copy(), G, None, U)


def cp_full(W, rng):
    cout, cin, k, _ = W.shape
    R = cin * k * k
    B = np.zeros((R, cin))
    Kv = np.zeros((R, k))
    Kh = np.zeros((R, k))
    A = np.zeros((cout, R))
    r = 0
    for i in range(cin):
        for a in range(k):
            for bb in range(k):
                B[r, i] = 1.0
                Kv[r, a] = 1.0
                Kh[r, bb] = 1.0
                A[:, r] = W[:, i, a, bb]
                r += 1
    return Decomp(1, "cp", R, R, B, Kv, Kh, A)


@pytest.mark.parametrize("cin,cout,k,s,p", [(4, 6, 3, 1, 1), (5, 3, 3, 2, 1), (3, 8, 7, 2, 3), (6, 6, 1, 2, 0)])
def test_tucker2_full_rank_reconstructs_conv(cin, cout, k, s, p):
    m, W, b = _single_conv_model(cin, cout, k, s, p, tucker_full)
    x = np.random.default_rng(3).standard_normal((2, m.height, m.width, cin))
    pl = oracle.plan(m)
    roles = [n.role for n in pl.graph.nodes]
    assert roles == ["", "fconv", "core", "lconv"]
    got = oracle.run_unfused(pl, x)
    np.testing.assert_allclose(got, _ref(m, W, b, x), rtol=1e-10, atol=1e-10)


@pytest.mark.parametrize("cin,cout,k,s,p", [(2, 5, 3, 1, 1), (3, 4, 3, 2, 1), (2, 3, 5, 2, 2), (3, 3, 3, 1, 0)])
def test_cp_full_rank_reconstructs_conv(cin, cout, k, s, p):
    m, W, b = _single_conv_model(cin, cout, k, s, p, cp_full)
    x = np.random.default_rng(4).standard_normal((2, m.height, m.width, cin))
    pl = oracle.plan(m)
    g = pl.graph
    assert [n.role for n in g.nodes] == ["", "fconv", "core", "core", "lconv"]
    assert (g.nodes[2].kh, g.nodes[2].kw, g.nodes[2].sh, g.nodes[2].ph) == (k, 1, s, p)
    assert (g.nodes[3].kh, g.nodes[3].kw, g.nodes[3].sw, g.nodes[3].pw) == (1, k, s, p)
    got = oracle.run_unfused(pl, x)
    np.testing.assert_allclose(got, _ref(m, W, b, x), rtol=1e-10, atol=1e-10)


def tt_full(W, rng):
    """TT-SVD (Oseledets' sequential truncated SVDs, no truncation) of W in mode order
    (C_in, K_h, K_w, C_out): exact TT ranks r1 = min(C_in, K K C_out),
    r2 = min(r1 K, K C_out), r3 = min(r2 K, C_out)."""
    cout, cin, k, _ = W.shape
    A = np.transpose(W, (1, 2, 3, 0))                               # [C_in, K_h, K_w, C_out]
    U1, S1, V1 = np.linalg.svd(A.reshape(cin, k * k * cout), full_matrices=False)
    r1 = len(S1)
    rest = (S1[:, None] * V1).reshape(r1 * k, k * cout)
    U2, S2, V2 = np.linalg.svd(rest, full_matrices=False)
    r2 = len(S2)
    rest = (S2[:, None] * V2).reshape(r2 * k, cout)
    U3, S3, V3 = np.linalg.svd(rest, full_matrices=False)
    r3 = len(S3)
    G1 = U1                                                         # [C_in, r1]
    G2 = U2.reshape(r1, k, r2)
    G3 = U3.reshape(r2, k, r3)
    G4 = S3[:, None] * V3                                           # [r3, C_out]
    # conv weights: fconv [r1, C_in]; K x 1 core [r2, r1, K]; 1 x K core [r3, r2, K]; lconv [C_out, r3]
    return Decomp(1, "tt", r1, r3, G1.T.copy(), np.transpose(G2, (2, 0, 1)).copy(),
                  np.transpose(G3, (2, 0, 1)).copy(), G4.T.copy(), rank_mid=r2)


@pytest.mark.parametrize("cin,cout,k,s,p", [(3, 5, 3, 1, 1), (4, 4, 3, 2, 1), (2, 3, 5, 2, 2), (3, 2, 3, 1, 0)])
def test_tt_full_rank_reconstructs_conv(cin, cout, k, s, p):
    """Tensor-Train (reading R33) at the exact TT ranks reproduces the conv, including
    stride and padding, through fconv -> K x 1 core -> 1 x K core -> lconv."""
    m, W, b = _single_conv_model(cin, cout, k, s, p, tt_full)
    x = np.random.default_rng(5).standard_normal((2, m.height, m.width, cin))
    pl = oracle.plan(m)
    g = pl.graph
    assert [n.role for n in g.nodes] == ["", "fconv", "core", "core", "lconv"]
    assert (g.nodes[2].kh, g.nodes[2].kw, g.nodes[2].sh, g.nodes[2].ph, g.nodes[2].groups) == (k, 1, s, p, 1)
    assert (g.nodes[3].kh, g.nodes[3].kw, g.nodes[3].sw, g.nodes[3].pw, g.nodes[3].groups) == (1, k, s, p, 1)
    d = m.decomps[1]
    assert (g.nodes[1].C, g.nodes[2].C, g.nodes[3].C) == (d.rank_in, d.rank_mid, d.rank_out)
    got = oracle.run_unfused(pl, x)
    np.testing.assert_allclose(got, _ref(m, W, b, x), rtol=1e-10, atol=1e-10)


def test_tt_truncated_ranks_change_the_output():
    """A TT train truncated below its exact ranks no longer reproduces the conv (the pin above
    is not vacuous: every core takes part)."""
    def tt_cut(W, rng):
        d = tt_full(W, rng)
        d.core = d.core.copy()
        d.core[-1] = 0.0                                            # drop one r2 channel
        return d
    m, W, b = _single_conv_model(3, 4, 3, 1, 1, tt_cut)
    x = np.random.default_rng(6).standard_normal((2, m.height, m.width, 3))
    got = oracle.run_unfused(oracle.plan(m), x)
    assert np.abs(got - _ref(m, W, b, x)).max() > 1e-3


def test_tucker2_omitted_factors_and_bias_placement():
    """R_in == C_in drops the fconv; R_out == C_out drops the lconv and the
    bias moves onto the core (O1)."""
    def no_last(W, rng):
        cout, cin = W.shape[:2]
        V = _orth(rng, cin)
        G = np.einsum("oikl,ib->obkl", W, V)
        return Decomp(1, "tucker2", cin, cout, V.T.copy(), G, None, None)

    m, W, b = _single_conv_model(4, 3, 3, 1, 1, no_last)
    pl = oracle.plan(m)
    assert [n.role for n in pl.graph.nodes] == ["", "fconv", "core"]
    assert pl.graph.nodes[2].bias is not None
    x = np.random.default_rng(5).standard_normal((2, m.height, m.width, 4))
    np.testing.assert_allclose(oracle.run_unfused(pl, x), _ref(m, W, b, x), rtol=1e-10, atol=1e-10)


@pytest.mark.parametrize("cin,cout,k,s,p", [(4, 6, 2, 2, 0), (5, 3, 3, 2, 1)])
def test_tucker2_full_rank_reconstructs_conv_transpose(cin, cout, k, s, p):
    """UNet up-conv: the Tucker-2 expansion fconv (V^T) -> transposed core
    G -> lconv (U) of a ConvTranspose2d weight W [C_in, C_out, k, k], with
    G[a, b] = sum_{c,o} V[c, a] W[c, o] U[o, b], reproduces torch's conv_transpose2d of W."""
    rng = np.random.default_rng(9)
    W = rng.standard_normal((cin, cout, k, k))
    b = rng.standard_normal(cout)
    U, V = _orth(rng, cout), _orth(rng, cin)
    G = np.einsum("ca,cokl,ob->abkl", V, W, U)
    m = Model("single_t", 2, 5, 4, cin, "f32")
    m.layers = [Layer("input", [], out_channels=cin),
                Layer("conv_transpose", [0], out_channels=cout, kernel=k, stride=s, pad=p, weight=W, bias=b)]
    m.decomps = {1: Decomp(1, "tucker2", cin, cout, V.T.copy(), G, None, U)}
    x = rng.standard_normal((2, 5, 4, cin))
    got = oracle.run_unfused(oracle.plan(m), x)
    t = F.conv_transpose2d(torch.from_numpy(np.transpose(x, (0, 3, 1, 2))), torch.from_numpy(W),
                           torch.from_numpy(b), stride=s, padding=p)
    np.testing.assert_allclose(got, np.transpose(t.numpy(), (0, 2, 3, 1)), rtol=1e-10, atol=1e-10)
