"""Cycle accounting of pair 0's MMA issuer and one epilogue warp for every tc_pair launch
(experiment build):
TEMCO_VARIANT=trace TEMCO_EXTRA_FLAGS="-DTEMCO_TRACE -DTEMCO_NOSTAMP" python -m paper_conf_icpp_songljkj0024_b200.build
TEMCO_LIB=build/exp/libtemco_trace.so python scripts/pair_prof.py [config]
"""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as W
from paper_conf_icpp_songljkj0024_b200 import Plan
import paper_conf_icpp_songljkj0024_b200.temco as T

cfg = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
m = W.build_config(cfg)
p = Plan(m)
d = p.describe()
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
buf = (ctypes.c_ulonglong * (64 * 16))()
T._lib.temco_debug_pair_dbg(int(os.environ.get("PAIR_DBG", "0")))
p.run(x, y); torch.cuda.synchronize()
ms = np.array(p.run_profiled(x, y))
T._lib.temco_debug_pair_prof(buf)
p.run(x, y); torch.cuda.synchronize()
n = T._lib.temco_debug_pair_prof(buf)
a = np.array(buf, dtype=np.float64).reshape(64, 16)
steps = [(i, s) for i, s in enumerate(d["steps"]) if s["kernel"] == "tc_pair"]
print(f"{n} pair launches; {len(steps)} pair steps")
print("  out    ms tiles U  D | issuer %: full accE  pF   oE  mma  com (cycles) | epi %: accF  pE   ld  math  oF   P   out (cycles)")
for k, (i, s) in enumerate(steps[:n]):
    r = a[k]
    t0, t8 = max(r[0], 1), max(r[8], 1)
    tc = s["tc"]
    print(f"{s['out']:5d} {ms[i]:.3f} {tc['ntiles']:5d} {tc['units']:2d} {tc['levels']:2d} | " +
          " ".join(f"{100 * r[j] / t0:4.1f}" for j in (1, 2, 3, 4, 5, 6)) + f" ({int(r[0])}) | " +
          " ".join(f"{100 * r[j] / t8:4.1f}" for j in (9, 10, 11, 12, 13, 14, 15)) + f" ({int(r[8])})")
