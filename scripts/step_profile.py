"""Per-step device time of a plan (CUDA events around every step)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as W
from paper_conf_icpp_songljkj0024_b200 import Plan
cfg = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
m = W.build_config(cfg)
p = Plan(m, flags=int(os.environ.get("TEMCO_PLAN_FLAGS", "0")))
d = p.describe()
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
for _ in range(3): p.run(x, y)
ms = np.zeros(len(d["steps"]))
for _ in range(5): ms += np.array(p.run_profiled(x, y))
ms /= 5
rows = []
for s, t in zip(d["steps"], ms):
    if s["kernel"] == "none": continue
    f = s.get("alg_flops", s["flops"]); b = s.get("alg_bytes", s["io_bytes"])
    rows.append((t, s["kernel"], s["out"], s["op"], s["role"], len(s["members"]), f / t / 1e9 if t else 0, b / t / 1e6 if t else 0))
rows.sort(reverse=True)
print(f"{cfg}: total {ms.sum():.3f} ms")
for r in rows[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print("%8.3f ms %-14s out=%-5d %-8s %-6s members=%-3d %8.1f TFLOP/s %8.1f GB/s" % r)
