"""The small parity cases of test_gpu_parity.py exercise every kernel family the
full-size bench configs launch (host-only: plans with TEMCO_FLAG_NO_DEVICE pick
the same kernels as device plans)."""
import collections

import workloads as W


def _kernels(m, flags=0):
    from paper_conf_icpp_songljkj0024_b200 import FLAG_NO_DEVICE, Plan
    p = Plan(m, flags=FLAG_NO_DEVICE | flags)
    return collections.Counter(s["kernel"] for s in p.describe()["steps"])


def test_small_cases_cover_the_full_configs():
    small = collections.Counter()
    for m in (W.resnet18_cifar(batch=3, dtype="bf16", height=16, width=16),
              W.resnet50(batch=2, dtype="bf16", height=64, width=64),
              W.vgg16_cp(batch=2, dtype="bf16", height=32, width=32),
              W.densenet121(batch=2, dtype="bf16", height=64, width=64),
              W.alexnet(batch=60, dtype="bf16", height=224, width=224),
              W.unet(batch=2, dtype="bf16", height=32, width=32, base=64),
              W.resnet18_cifar(batch=3, dtype="bf16", height=16, width=16, tt=True)):
        small.update(_kernels(m))
    full = collections.Counter()
    for name in ("resnet18_cifar", "resnet50", "vgg16_cp", "densenet121", "alexnet", "unet", "resnet18_tt"):
        full.update(_kernels(W.build_config(name)))
    assert set(full) <= set(small), set(full) - set(small)
    # the tensor-core families are all on the bench path
    for k in ("tc_chain", "tc_pair", "mma_lean", "mma_conv_tile", "mma_conv_stem", "tc_conv", "tc_gemm",
              "tc_gemm_convt"):
        assert full[k] > 0, k


def test_opt_in_concat_kernel_is_selected_by_its_flag():
    from paper_conf_icpp_songljkj0024_b200 import FLAG_MMA_CAT
    m = W.densenet121(batch=2, dtype="bf16", height=64, width=64)
    assert _kernels(m)["mma_cat"] == 0
    assert _kernels(m, FLAG_MMA_CAT)["mma_cat"] > 0


def test_bf16_full_configs_never_fall_back_to_the_interpreter():
    """Every fused group of the bench configs lowers to a tensor-core kernel: a lowering
    regression would silently route a group to the SIMT interpreter (correct, 100x slower)."""
    for name in ("resnet18_cifar", "resnet50", "vgg16_cp", "densenet121"):
        ks = _kernels(W.build_config(name))
        assert ks["simt_group"] == 0 and ks["simt_group_gap"] == 0, (name, ks)


def _silu(m):
    for layer in m.layers:
        if layer.op == "relu":
            layer.op = "silu"
    return m


def test_silu_full_configs_on_tensor_core_kernels():
    """SiLU plans of the bench configs (bench.py --act silu) lower every fused group to
    a tensor-core kernel, like the ReLU plans; the small SiLU parity cases of
    test_gpu_ablation.py cover the kernel families they launch."""
    small = collections.Counter()
    for m in (W.resnet18_cifar(batch=2, dtype="bf16", height=16, width=16),
              W.resnet50(batch=2, dtype="bf16", height=64, width=64),
              W.densenet121(batch=2, dtype="bf16", height=64, width=64)):
        small.update(_kernels(_silu(m)))
    for name in ("resnet18_cifar", "resnet50", "vgg16_cp", "densenet121"):
        k = _kernels(_silu(W.build_config(name)))
        assert not any(x.startswith("simt_group") for x in k), (name, k)
        if name != "vgg16_cp":
            assert set(k) <= set(small), (name, set(k) - set(small))
