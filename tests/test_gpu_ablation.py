"""GPU parity for the paper's ablation variants and the SiLU activation
(SURVEY 8(f) rows f2/f3).

* Ablations (Fig. 10/11): "Decomposed" = no skip optimization and no
  fusion, "Fusion only" = TEMCO_FLAG_NO_SKIPOPT, "Skip-Opt only" =
  TEMCO_FLAG_NO_FUSION.  Each GPU plan is compared with the oracle's executor
  of the same ablated plan (oracle.plan(m, skip_opt=..., fusion=...)) and with
  the op-by-op decomposed execution, and its peak internal bytes with the
  oracle's.
* SiLU (P:L307 names ReLU and SiLU as the fusable activations): the same small
  graphs with every ReLU replaced by SiLU; fp32 and bf16 bars as
  test_gpu_parity.
"""
import copy

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


def _run(m, flags, x):
    from paper_conf_icpp_songljkj0024_b200 import Plan
    p = Plan(m, flags=flags)
    xt = torch.from_numpy(x).cuda().to(torch.bfloat16 if m.dtype == "bf16" else torch.float32)
    y = torch.full(p.output_shape(), float("nan"), dtype=torch.float32, device="cuda")
    p.run(xt, y, None)
    torch.cuda.synchronize()
    return p, y.cpu().numpy().astype(np.float64)


def _rel(a, b):
    return float(np.linalg.norm(a - b) / np.linalg.norm(b))


GRAPHS = {
    "c1": lambda dt: W.c1_basic_block(dtype=dt, batch=2),
    "t2_3": lambda dt: W.t2_stem_blocks(3, dtype=dt, batch=2),
    "t3": lambda dt: W.t3_mini_bottleneck(dtype=dt, batch=2),
    "t4": lambda dt: W.t4_mini_densenet(dtype=dt, batch=2),
    "resnet18_s": lambda dt: W.resnet18_cifar(batch=2, dtype=dt, height=16, width=16),
    "densenet121_s": lambda dt: W.densenet121(batch=2, dtype=dt, height=64, width=64),
    "resnet50_s": lambda dt: W.resnet50(batch=2, dtype=dt, height=64, width=64),
}
TOL = {"f32": 1e-4, "bf16": 2e-2}


def _variants():
    from paper_conf_icpp_songljkj0024_b200 import FLAG_NO_FUSION, FLAG_NO_SKIPOPT
    return {"decomposed": (FLAG_NO_FUSION | FLAG_NO_SKIPOPT, dict(skip_opt=False, fusion=False)),
            "fusion_only": (FLAG_NO_SKIPOPT, dict(skip_opt=False)),
            "skipopt_only": (FLAG_NO_FUSION, dict(fusion=False))}


@pytest.mark.parametrize("dt", ["f32", "bf16"])
@pytest.mark.parametrize("name", list(GRAPHS))
def test_ablation_variants(name, dt):
    m = GRAPHS[name](dt)
    x = W.make_input(m)
    ref_dec = oracle.run_unfused(oracle.plan(m), x)
    for vname, (flags, okw) in _variants().items():
        o = oracle.plan(m, **okw)
        ref = oracle.run_temco(o, x)
        p, y = _run(m, flags, x)
        assert y.shape == ref.shape
        assert np.isfinite(y).all(), vname
        assert _rel(y, ref) <= TOL[dt], (vname, _rel(y, ref))
        assert _rel(y, ref_dec) <= TOL[dt], (vname, _rel(y, ref_dec))
        assert p.peak_internal_bytes(0) == o.peak_fused, vname


def _silu(m):
    m = copy.deepcopy(m)
    n = 0
    for layer in m.layers:
        if layer.op == "relu":
            layer.op = "silu"
            n += 1
    assert n > 0
    return m


@pytest.mark.parametrize("dt", ["f32", "bf16"])
@pytest.mark.parametrize("name", ["c1", "t3", "t4", "resnet18_s", "resnet50_s", "densenet121_s"])
def test_silu_activation(name, dt):
    from paper_conf_icpp_songljkj0024_b200 import FLAG_NO_FUSION
    m = _silu(GRAPHS[name](dt))
    x = W.make_input(m)
    o = oracle.plan(m)
    ref = oracle.run_temco(o, x)
    # SiLU is not ReLU: the plan must not silently compute max(x, 0)
    relu_ref = oracle.run_temco(oracle.plan(GRAPHS[name](dt)), x)
    assert _rel(ref, relu_ref) > 10 * TOL[dt]
    if dt == "bf16" and name in ("resnet18_s", "resnet50_s", "densenet121_s"):
        from paper_conf_icpp_songljkj0024_b200 import FLAG_NO_DEVICE, Plan
        kernels = {s["kernel"] for s in Plan(m, flags=FLAG_NO_DEVICE).describe()["steps"]}
        assert kernels & {"mma_lean", "mma_chain"} and kernels & {"tc_chain", "tc_chain_wide"}, kernels   # SiLU on the tensor-core kernels
        assert not any(k.startswith("simt_group") for k in kernels), kernels            # incl. pooled members
    for flags in (0, FLAG_NO_FUSION):
        p, y = _run(m, flags, x)
        assert np.isfinite(y).all()
        assert _rel(y, ref) <= TOL[dt], (flags, _rel(y, ref))
    assert p.peak_internal_bytes(1) == o.peak_unfused


@pytest.mark.parametrize("name", ["t4", "resnet18_s", "densenet121_s"])
def test_vectorised_elementwise_bit_exact(name, monkeypatch):
    """The 16-byte elementwise kernel (standalone BN / ReLU / add / concat / pools of
    unfused plans) does the scalar kernel's arithmetic: identical bits."""
    from paper_conf_icpp_songljkj0024_b200 import FLAG_NO_FUSION, FLAG_NO_SKIPOPT
    m = GRAPHS[name]("bf16")
    x = W.make_input(m)
    _, y_vec = _run(m, FLAG_NO_FUSION | FLAG_NO_SKIPOPT, x)
    monkeypatch.setenv("TEMCO_NO_EW_VEC", "1")
    _, y_ref = _run(m, FLAG_NO_FUSION | FLAG_NO_SKIPOPT, x)
    assert np.array_equal(y_vec, y_ref)
