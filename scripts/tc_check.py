"""Quick GPU check of the fused-group kernel paths vs the oracle."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as W, oracle
from paper_conf_icpp_songljkj0024_b200 import Plan, FLAG_SIMT_ONLY, FLAG_MMA_SMALL

def run(m, flags, x):
    p = Plan(m, flags=flags)
    xt = torch.from_numpy(x).cuda().to(torch.bfloat16)
    y = torch.full(p.output_shape(), float('nan'), device='cuda')
    p.run(xt, y); torch.cuda.synchronize()
    return p, y.cpu().numpy()

rel = lambda a, b: float(np.linalg.norm(a - b) / np.linalg.norm(b))
cases = [W.t2_stem_blocks(3, dtype='bf16', batch=3), W.resnet18_cifar(batch=3, dtype='bf16', height=16, width=16),
         W.resnet50(batch=2, dtype='bf16', height=64, width=64), W.vgg16_cp(batch=2, dtype='bf16', height=32, width=32),
         W.densenet121(batch=2, dtype='bf16', height=64, width=64)]
for m in cases:
    x = W.make_input(m)
    ref = oracle.run_temco(oracle.plan(m), x)
    p, y = run(m, 0, x)
    _, yt = run(m, FLAG_MMA_SMALL, x)
    _, ys = run(m, FLAG_SIMT_ONLY, x)
    kinds = {}
    for s in p.describe()["steps"]:
        kinds[s["kernel"]] = kinds.get(s["kernel"], 0) + 1
    print(m.name, "default %.3e" % rel(y, ref), "mma-small %.3e" % rel(yt, ref), "simt %.3e" % rel(ys, ref),
          "finite", bool(np.isfinite(y).all()), kinds, flush=True)
