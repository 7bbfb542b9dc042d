"""ResNet-50 stem pooled group in isolation (lconv 8->64, BN, ReLU, maxpool 3x3 s2, fconv): profiling target."""
import sys, os
sys.path.insert(0, os.getcwd())
import torch
import workloads as W
from workloads.models import _G
from paper_conf_icpp_songljkj0024_b200 import Plan
g = _G("pool", 256, 112, 112, 8, "bf16", 3, rank=lambda c: 8)
a = g.maxpool(g.relu(g.bn(g.conv(0, 64, 1, name="c0"))), 3, 2, 1)
g.conv(a, 64, 1, name="c1")
m = g.m
p = Plan(m)
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
p.run(x, y); torch.cuda.synchronize()
print([ (s["kernel"], round(t,3)) for s, t in zip(p.describe()["steps"], p.run_profiled(x, y))])
