"""Planner (C++, libtemco.so) vs oracle (Python): identical rewrite, schedule
and bit-exact peak internal bytes on every config at full size.

Host-only: plans are created with TEMCO_FLAG_NO_DEVICE, so no GPU is needed.
"""
import pytest

import oracle
import workloads as W
from paper_conf_icpp_songljkj0024_b200 import (FLAG_NO_DEVICE, FLAG_NO_FUSION, FLAG_NO_SKIPOPT,
                                              FLAG_OVERHEAD_NEVER, FLAG_PAPER_SCHEDULE, Plan, TemcoError)

KEYS = ("kind", "out", "op", "role", "members", "inputs", "bytes", "extra")

SMALL = {
    "c1": W.c1_basic_block, "t1": W.t1_chain, "t2_1": lambda: W.t2_stem_blocks(1),
    "t2_3": lambda: W.t2_stem_blocks(3), "t3": W.t3_mini_bottleneck, "t4": W.t4_mini_densenet,
    "c1_bf16": lambda: W.c1_basic_block(dtype="bf16", batch=3),
}
FULL = ["resnet18_cifar", "resnet50", "vgg16_cp", "densenet121", "alexnet", "unet", "resnet18_tt"]


def _compare(m, flags=0, **okw):
    p = Plan(m, flags=FLAG_NO_DEVICE | flags)
    o = oracle.plan(m, **okw)
    d = p.describe()
    assert p.peak_internal_bytes(0) == o.peak_fused
    assert p.peak_internal_bytes(1) == o.peak_unfused
    assert d["O"] == o.O
    assert [{k: s[k] for k in KEYS} for s in d["steps"]] == o.describe()
    assert [s["live"] for s in d["steps"]] == o.live_fused
    assert d["live_unfused"] == o.live_unfused
    dec = [(x["kind"], x["node"]) + ((x["list"],) if x["kind"] == "skip-optimized" else ()) for x in d["decisions"]]
    assert dec == [tuple(e) for e in o.log]
    return p, o


@pytest.mark.parametrize("name", list(SMALL))
def test_small_graphs(name):
    _compare(SMALL[name]())


@pytest.mark.parametrize("name", FULL)
def test_full_configs(name):
    m = W.build_config(name)
    p, o = _compare(m)
    # the north-star >= 70 % target is stated for the BASELINE.json configs; AlexNet (f2, no
    # skip connections: activation-layer fusion only, P:L355 reports 49.4 %) reaches 54.9 %
    assert 1 - p.peak_internal_bytes(0) / p.peak_internal_bytes(1) >= (0.54 if name == "alexnet" else 0.70)


@pytest.mark.parametrize("name", FULL + list(SMALL))
def test_paper_schedule_mode(name):
    """TEMCO_FLAG_PAPER_SCHEDULE == the oracle without readings R34 / R35 (the paper's own
    schedule, whose peaks SURVEY P2 pins)."""
    m = W.build_config(name) if name in FULL else SMALL[name]()
    _compare(m, FLAG_PAPER_SCHEDULE, cp_pair=False, fold_cores=False, pool_first=False, cse=False, reorder=False)


@pytest.mark.parametrize("name", ["t2_3", "t3", "t4"])
def test_ablations(name):
    m = SMALL[name]()
    _compare(m, FLAG_NO_FUSION, fusion=False)
    _compare(m, FLAG_NO_SKIPOPT, skip_opt=False)
    _compare(m, FLAG_OVERHEAD_NEVER, policy="never")


def test_distance_threshold():
    m = W.t2_stem_blocks(2)
    p = Plan(m, flags=FLAG_NO_DEVICE, distance_threshold=100)
    o = oracle.plan(m, distance_threshold=100)
    assert p.peak_internal_bytes(0) == o.peak_fused == o.peak_unfused


def test_rejects_bad_graphs():
    m = W.c1_basic_block()
    with pytest.raises(TemcoError) as e:
        Plan(m, flags=FLAG_NO_DEVICE, skip_edges=[])          # declared skip edges must match
    assert e.value.status == 2
    m.layers[2].inputs = [5]                                  # non-topological input
    with pytest.raises(TemcoError) as e:
        Plan(m, flags=FLAG_NO_DEVICE, skip_edges=[])
    assert e.value.status == 2
    m = W.c1_basic_block()
    m.decomps[1].rank_in = 0
    with pytest.raises(TemcoError) as e:
        Plan(m, flags=FLAG_NO_DEVICE)
    assert e.value.status == 3


def test_no_device_plan_refuses_to_run():
    p = Plan(W.c1_basic_block(), flags=FLAG_NO_DEVICE)
    with pytest.raises(TemcoError) as e:
        p.run(1, 1, stream=0)
    assert e.value.status == 7


@pytest.mark.parametrize("name", ["c1", "t3", "t4"])
def test_silu_plans(name):
    """SiLU is fusable like ReLU -- same rewrite, groups and peak bytes."""
    import copy
    m = copy.deepcopy(SMALL[name]())
    for layer in m.layers:
        if layer.op == "relu":
            layer.op = "silu"
    p, o = _compare(m)
    assert any(s["kind"] == "group" and "silu" in s["op"] for s in p.describe()["steps"]) or \
        any(st.kind == "group" for st in o.steps)


@pytest.mark.parametrize("name", FULL + ["t3", "t4"])
def test_step_flops_match_oracle(name):
    """The C++ planner's per-node FLOP counts (node_flops, reading R1) equal the
    oracle's graph.flops for every node of every schedule step (the numbers
    Overhead compares; graph.flops itself is pinned by hand counts in
    test_oracle_flops.py)."""
    from oracle.graph import flops
    m = W.build_config(name) if name in FULL else SMALL[name]()
    p = Plan(m, flags=FLAG_NO_DEVICE)
    o = oracle.plan(m)
    g = o.graph
    nodes = dict(g.nodes_by_id)
    nodes.update(o.onodes)
    g2 = type(g)(nodes=g.nodes, output=g.output, batch=g.batch, dtype=g.dtype, orig_flops=g.orig_flops,
                 nodes_by_id=nodes)
    for s in p.describe()["steps"]:
        want = sum(flops(g2, nodes[i]) for i in s["members"] if nodes[i].op != "input")
        assert s["flops"] == want, (name, s["out"], s["flops"], want)
