"""Executors (oracle step O11): the unfused decomposed model and the
TeMCO-transformed model, both in fp64.

TeMCO preserves the semantics of the decomposed model, so the
two must agree to rounding; the TeMCO executor runs the schedule S with only
the tensors S materialises: a fused group is evaluated from its root down its
member expression tree using nothing but its declared group inputs (reduced
tensors, plus external full tensors), and every tensor is dropped right after
the last step that reads it -- reading a dropped or undeclared tensor raises.
"""
from __future__ import annotations

import numpy as np

from . import ops
from .graph import Node


def apply(v: Node, xs):
    """One node of L / O on its input tensors (NHWC fp64)."""
    if v.op == "conv":
        return ops.conv2d(xs[0], v.weight, v.bias, (v.sh, v.sw), (v.ph, v.pw), v.groups)
    if v.op == "convt":
        return ops.conv_transpose2d(xs[0], v.weight, v.bias, v.sh, v.ph)
    if v.op == "bn":
        g, b, m, var, eps = v.bn
        return ops.batchnorm(xs[0], g, b, m, var, eps)
    if v.op == "relu":
        return ops.relu(xs[0])
    if v.op == "silu":
        return ops.silu(xs[0])
    if v.op == "add":
        return ops.add(xs)
    if v.op == "concat":
        return ops.concat(xs)
    if v.op == "maxpool":
        return ops.maxpool(xs[0], v.kh, v.sh, v.ph)
    if v.op == "avgpool":
        return ops.avgpool(xs[0], v.kh, v.sh)
    if v.op == "gap":
        return ops.gap(xs[0])
    if v.op == "linear":
        return ops.linear(xs[0], v.weight, v.bias)
    raise ValueError(v.op)


def _as_output(y):
    """[N,1,1,K] (GAP / linear outputs) -> [N,K]; feature maps stay NHWC."""
    if y.ndim == 4 and y.shape[1] == 1 and y.shape[2] == 1:
        return y.reshape(y.shape[0], -1)
    return y


def run_decomposed_order(nodes, output, x, node_map=None):
    """Run a node list op by op, materialising every tensor."""
    node_map = node_map or {n.id: n for n in nodes}
    env = {nodes[0].id: np.asarray(x, np.float64)}
    for nid in (n.id if isinstance(n, Node) else n for n in nodes[1:]):
        v = node_map[nid]
        env[nid] = apply(v, [env[i] for i in v.inputs])
    return _as_output(env[output])


def run_unfused(plan, x):
    """The paper's "Decomposed" baseline: L executed op by op."""
    g = plan.graph
    return run_decomposed_order(g.nodes, g.output, x)


def _eval_group(plan, step, env):
    """Every output of a fused group (its root; a merged group's further reduce outputs,
    reading R37, share the one evaluation of the restored tensor)."""
    members = set(step.members)
    memo = {}

    def value(nid):
        if nid in memo:
            return memo[nid]
        if nid not in members:
            if nid not in step.inputs:
                raise RuntimeError(f"group {step.out} reads undeclared tensor {nid}")
            return env[nid]                      # KeyError if already dropped
        v = plan.onodes[nid]
        memo[nid] = apply(v, [value(i) for i in v.inputs])
        return memo[nid]

    return {o: value(o) for o in step.outs}


def run_step(plan, t, env, which=None):
    """Output `which` (default: the step's root) of schedule step t of S given its input
    tensors env[id] (per-step parity tests feed the GPU's own inputs, so each step is
    checked in isolation)."""
    s = plan.steps[t]
    if s.kind == "group":
        return _eval_group(plan, s, env)[s.out if which is None else which]
    v = plan.onodes[s.out]
    return apply(v, [env[i] for i in v.inputs])


def run_temco(plan, x, on_step=None, on_tensor=None):
    """Run the TeMCO schedule S (fused groups + remaining ops).  on_step(t, tensor),
    if given, sees every step's output as it is produced, on_tensor(id, tensor) every
    tensor a step defines (a merged group defines several; per-step parity tests)."""
    g = plan.graph
    steps = plan.steps
    last = {}
    for t, s in enumerate(steps):
        for i in s.inputs:
            last[i] = t
    env = {}
    for t, s in enumerate(steps):
        if t == 0:
            env[s.out] = np.asarray(x, np.float64)
        elif s.kind == "group":
            env.update(_eval_group(plan, s, env))
        else:
            v = plan.onodes[s.out]
            env[s.out] = apply(v, [env[i] for i in v.inputs])
        if on_step is not None:
            on_step(t, env[s.out])
        if on_tensor is not None:
            for o in s.outs:
                on_tensor(o, env[o])
        for i in s.inputs:
            if last[i] == t and i != g.output:
                del env[i]
    return _as_output(env[g.output])
