"""One small TeMCO inference for compute-sanitizer (memcheck / racecheck / synccheck).
usage: compute-sanitizer --tool <tool> python scripts/sanitize_run.py <graph> [flags]
Graphs cover every kernel family: c1 (fp32 SIMT), t2_3 / t3 / t4 (bf16 small graphs),
resnet50_s (tc_pair, tc_chain, mma_* kernels, GAP root), vgg16_s (CP depthwise,
tc_gemm split-K head), alexnet_s (11x11 stride-4 stem, tc_gemm)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import workloads as W
from paper_conf_icpp_songljkj0024_b200 import Plan

GRAPHS = {
    "c1": lambda: W.c1_basic_block(dtype="f32", batch=2),
    "t2_3": lambda: W.t2_stem_blocks(3, dtype="bf16", batch=3),
    "t3": lambda: W.t3_mini_bottleneck(dtype="bf16", batch=2),
    "t4": lambda: W.t4_mini_densenet(dtype="bf16", batch=2),
    "resnet50_s": lambda: W.resnet50(batch=2, dtype="bf16", height=64, width=64),
    "vgg16_s": lambda: W.vgg16_cp(batch=2, dtype="bf16", height=32, width=32),
    "alexnet_s": lambda: W.alexnet(batch=2, dtype="bf16", height=127, width=127),
}
m = GRAPHS[sys.argv[1]]()
flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
p = Plan(m, flags=flags)
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16 if m.dtype == "bf16" else torch.float32)
y = torch.empty(p.output_shape(), dtype=torch.float32, device="cuda")
p.run(x, y)
torch.cuda.synchronize()
assert np.isfinite(y.cpu().numpy()).all()
kernels = sorted({s["kernel"] for s in p.describe()["steps"]} - {"none"})
print(sys.argv[1], "ok:", " ".join(kernels))
