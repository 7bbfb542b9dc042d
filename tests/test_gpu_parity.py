"""GPU parity: temco_run (through the C ABI) vs the fp64 oracle.

Bars (BASELINE.json north star): relative L2 <= 1e-4 in fp32 mode (SIMT
kernels, no TF32) and <= 2e-2 in bf16 mode (bf16 storage, fp32 accumulation;
the workloads hand both sides the same bf16-representable weights and input).
Peak internal bytes must equal the oracle's exactly.  Full-size configs run in
the launch configuration bench.py times; the oracle checks sampled images
(images are independent, the kernels batch-invariant).
"""
import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


def _plan_and_run(m, flags=0, x=None, stream=None):
    from paper_conf_icpp_songljkj0024_b200 import Plan
    p = Plan(m, flags=flags)
    if x is None:
        x = W.make_input(m)
    xt = torch.from_numpy(x).cuda().to(torch.bfloat16 if m.dtype == "bf16" else torch.float32)
    y = torch.full(p.output_shape(), float("nan"), dtype=torch.float32, device="cuda")
    p.run(xt, y, stream)
    torch.cuda.synchronize()
    return p, y.cpu().numpy().astype(np.float64)


def _rel(a, b):
    return float(np.linalg.norm(a - b) / np.linalg.norm(b))


SMALL = {
    "c1": lambda dt: W.c1_basic_block(dtype=dt, batch=2),
    "t1": lambda dt: W.t1_chain(dtype=dt, batch=2),
    "t2_1": lambda dt: W.t2_stem_blocks(1, dtype=dt, batch=2),
    "t2_3": lambda dt: W.t2_stem_blocks(3, dtype=dt, batch=3),
    "t3": lambda dt: W.t3_mini_bottleneck(dtype=dt, batch=2),
    "t4": lambda dt: W.t4_mini_densenet(dtype=dt, batch=2),
    "resnet18_s": lambda dt: W.resnet18_cifar(batch=3, dtype=dt, height=16, width=16),
    "resnet50_s": lambda dt: W.resnet50(batch=2, dtype=dt, height=64, width=64),
    "vgg16_s": lambda dt: W.vgg16_cp(batch=2, dtype=dt, height=32, width=32),
    "densenet121_s": lambda dt: W.densenet121(batch=2, dtype=dt, height=64, width=64),
    # batch 60 at 224: the 13x13 pooled group has enough pixels (10140, a ragged 256-pixel
    # pair tile) for the CTA-pair kernel, as at the full batch
    "alexnet_s": lambda dt: W.alexnet(batch=60, dtype=dt, height=224, width=224),
    # full width (base 64): the 3x3 cores of the bottom level exceed one SMEM weight block
    # (output-channel-sliced tc_conv), as in the full config
    "unet_s": lambda dt: W.unet(batch=2, dtype=dt, height=32, width=32, base=64),
    # Tensor-Train (f4): K x 1 and 1 x K cores on reduced channels
    "resnet18_tt_s": lambda dt: W.resnet18_cifar(batch=3, dtype=dt, height=16, width=16, tt=True),
}


@pytest.mark.parametrize("name", list(SMALL))
def test_fp32_mode(name):
    m = SMALL[name]("f32")
    x = W.make_input(m)
    p, y = _plan_and_run(m, x=x)
    o = oracle.plan(m)
    ref = oracle.run_temco(o, x)
    assert y.shape == ref.shape
    assert np.isfinite(y).all()
    assert _rel(y, ref) <= 1e-4, _rel(y, ref)
    assert p.peak_internal_bytes(0) == o.peak_fused and p.peak_internal_bytes(1) == o.peak_unfused


@pytest.mark.parametrize("name", list(SMALL))
def test_bf16_mode(name):
    from paper_conf_icpp_songljkj0024_b200 import FLAG_MMA_CAT, FLAG_MMA_SMALL, FLAG_SIMT_ONLY
    m = SMALL[name]("bf16")
    x = W.make_input(m)
    ref = oracle.run_temco(oracle.plan(m), x)
    for flags in (0, FLAG_SIMT_ONLY, FLAG_MMA_SMALL, FLAG_MMA_CAT):
        p, y = _plan_and_run(m, flags=flags, x=x)
        assert np.isfinite(y).all()
        assert _rel(y, ref) <= 2e-2, (flags, _rel(y, ref))


def test_ragged_batch_and_tiles():
    """batch / pixel counts that leave ragged tails in every kernel's tiling."""
    m = W.resnet18_cifar(batch=5, dtype="bf16", height=12, width=20)
    x = W.make_input(m)
    _, y = _plan_and_run(m, x=x)
    ref = oracle.run_temco(oracle.plan(m), x)
    assert _rel(y, ref) <= 2e-2


FULL = {"resnet18_cifar": [0, 77, 127], "resnet50": [0, 255], "vgg16_cp": [0, 255], "densenet121": [0, 127],
        "alexnet": [0, 255], "unet": [0, 15], "resnet18_tt": [0, 127]}


@pytest.mark.parametrize("name", list(FULL))
def test_full_config_sampled(name):
    """Full BASELINE.json config in the bench launch configuration; sampled
    images checked against the oracle one by one."""
    m = W.build_config(name)
    x = W.make_input(m)
    p, y = _plan_and_run(m, x=x)
    assert np.isfinite(y).all()
    o = oracle.plan(m)
    assert p.peak_internal_bytes(0) == o.peak_fused and p.peak_internal_bytes(1) == o.peak_unfused
    for i in FULL[name]:
        ref = oracle.run_temco(o, x[i:i + 1])
        assert _rel(y[i:i + 1], ref) <= 2e-2, (i, _rel(y[i:i + 1], ref))


def test_batch_invariance_and_shard_equivalence():
    """A shard (images 2..5 run as their own batch) reproduces the same rows of
    the full-batch run bit for bit: what the multi-GPU batch split relies on."""
    m = W.resnet50(batch=8, dtype="bf16", height=64, width=64)
    x = W.make_input(m)
    _, y = _plan_and_run(m, x=x)
    ms = W.resnet50(batch=4, dtype="bf16", height=64, width=64)
    _, ys = _plan_and_run(ms, x=x[2:6])
    assert np.array_equal(y[2:6], ys)


def test_cuda_graph_host_run_and_profiled_agree():
    from paper_conf_icpp_songljkj0024_b200 import FLAG_CUDA_GRAPH, Plan
    m = W.resnet18_cifar(batch=4, dtype="bf16")
    x = W.make_input(m)
    _, y0 = _plan_and_run(m, x=x)
    p = Plan(m, flags=FLAG_CUDA_GRAPH)
    xt = torch.from_numpy(x).cuda().to(torch.bfloat16)
    y = torch.empty(p.output_shape(), device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3):
            p.run(xt, y, s)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy(), y0)
    xh = torch.from_numpy(x).to(torch.bfloat16).pin_memory()
    yh = torch.empty(p.output_shape()).pin_memory()
    p.run_host(xh, yh, s)
    assert np.array_equal(yh.numpy(), y0)
    ms = p.run_profiled(xt, y, s)
    assert len(ms) == len(p.describe()["steps"]) and all(t >= 0 for t in ms)
    assert np.array_equal(y.cpu().numpy(), y0)


def test_device_mismatch_and_errors():
    from paper_conf_icpp_songljkj0024_b200 import Plan, TemcoError
    p = Plan(W.c1_basic_block(dtype="f32"))
    with pytest.raises(TemcoError) as e:
        p.run(0, 0, 0)
    assert e.value.status == 1


def test_run_host_async_pipeline_matches_device_run():
    """temco_run_host_async: consecutive calls alternate staging buffers and
    overlap the next input copy with the current run; every output equals the
    device-buffer run of the same input."""
    from paper_conf_icpp_songljkj0024_b200 import Plan
    m = W.resnet18_cifar(batch=4, dtype="bf16")
    xs = [W.make_input(m, start=4 * k, count=4) for k in range(3)]
    p = Plan(m)
    refs = [_plan_and_run(m, x=x)[1] for x in xs]
    s = torch.cuda.Stream()
    xh = [torch.from_numpy(x).to(torch.bfloat16).pin_memory() for x in xs]
    yh = [torch.empty(p.output_shape()).pin_memory() for _ in xs]
    for k in range(3):
        p.run_host_async(xh[k], yh[k], s)
    s.synchronize()
    for k in range(3):
        assert np.array_equal(yh[k].numpy(), refs[k])


def test_fp32_resnet18c_survey_parity_case():
    """SURVEY 8(d) C2 fp32 parity case: ResNet-18 (CIFAR) at 32x32, batch 8, fp32 mode
    (SIMT kernels, no TF32) within 1e-4 relative L2 of the fp64 oracle."""
    m = W.resnet18_cifar(batch=8, dtype="f32", height=32, width=32)
    x = W.make_input(m)
    p, y = _plan_and_run(m, x=x)
    o = oracle.plan(m)
    ref = oracle.run_temco(o, x)
    assert np.isfinite(y).all()
    assert _rel(y, ref) <= 1e-4, _rel(y, ref)
    assert p.peak_internal_bytes(0) == o.peak_fused


@pytest.mark.parametrize("name", ["t3", "resnet18_s", "resnet50_s", "resnet18_tt_s"])
@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_merge_and_reschedule_variants(name, dt):
    """Readings R37 (merged fconvs) and R38 (re-scheduling) under each policy: the default, the
    "bound" merge policy (every candidate merged: ResNet-50's stage-2 group on the CTA-pair kernel
    with two reduce outputs), and neither.  Output vs the oracle's plan with the same options, peak
    bytes exact; a merged group's outputs are checked step by step in test_gpu_steps.py."""
    from paper_conf_icpp_songljkj0024_b200 import FLAG_CSE_BOUND, FLAG_NO_CSE, FLAG_NO_RESCHEDULE
    m = SMALL[name](dt)
    x = W.make_input(m)
    tol = 1e-4 if dt == "f32" else 2e-2
    for flags, kw in ((0, {}), (FLAG_CSE_BOUND, {"cse_policy": "bound"}),
                      (FLAG_NO_CSE | FLAG_NO_RESCHEDULE, {"cse": False, "reorder": False})):
        o = oracle.plan(m, **kw)
        ref = oracle.run_temco(o, x)
        p, y = _plan_and_run(m, flags=flags, x=x)
        assert np.isfinite(y).all()
        assert _rel(y, ref) <= tol, (flags, _rel(y, ref))
        assert p.peak_internal_bytes(0) == o.peak_fused
        assert [s["extra"] for s in p.describe()["steps"]] == [s.extra for s in o.steps]
