"""One ResNet-50 b256 forward without CUDA graphs (ncu target)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as W
from paper_conf_icpp_songljkj0024_b200 import Plan
cfg = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
m = W.build_config(cfg)
p = Plan(m, flags=int(os.environ.get("TEMCO_PLAN_FLAGS", "0")))
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
p.run(x, y)
torch.cuda.synchronize()
print("done")
