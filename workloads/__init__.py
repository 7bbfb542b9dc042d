"""Seeded synthetic workloads shared by the oracle, the tests and bench.py.

This package holds ONLY input generation: layer graphs of the original
(undecomposed) models, randomly initialised decomposition factors, BN
statistics and images.  It contains none of the method's arithmetic (no
decomposition expansion, liveness, rewrite, fusion or convolution); both the
oracle (`oracle/`) and the product path (`paper_conf_icpp_songljkj0024_b200`)
consume what it produces, independently.
"""
from .models import (  # noqa: F401
    Layer, Decomp, Model, rank_rule, bf16_round, skip_edges, make_input,
    c1_basic_block, t1_chain, t2_stem_blocks, t3_mini_bottleneck, t4_mini_densenet,
    resnet18_cifar, resnet50, vgg16_cp, densenet121, alexnet, unet, CONFIGS, build_config,
)
