"""CTA-0 pipeline trace of one fused-group kernel (experiment build).

TEMCO_VARIANT=trace TEMCO_EXTRA_FLAGS=-DTEMCO_TRACE python -m paper_conf_icpp_songljkj0024_b200.build
TEMCO_LIB=build/exp/libtemco_trace.so TEMCO_TC_TRACE_OUT=<out id> python scripts/trace_group.py [config]
Rows (ns from the first stamp): 0 producer A issued, 1 MMA A ready, 2 MMA slot
free, 3 MMA slot committed, 4 team-0 acc ready, 5 team-0 slot released, 6 team-0
P written, 7 GEMM2 P ready, 8 GEMM2 P committed, 9 team-0 out ready, 10 team-1
acc ready, 11 GEMM2 out buffer free.
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
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
buf = (ctypes.c_longlong * (12 * 512))()
p.run(x, y)
torch.cuda.synchronize()
T._lib.temco_debug_trace(buf)   # clear
p.run(x, y)
torch.cuda.synchronize()
T._lib.temco_debug_trace(buf)
a = np.array(buf, dtype=np.int64).reshape(12, 512)
t0 = min(v for v in a.flatten() if v)
names = ["prod_A_issued", "mma_A_ready", "mma_slot_free", "mma_slot_commit", "t0_acc_ready", "t0_slot_release",
         "t0_P_written", "g2_P_ready", "g2_P_commit", "t0_out_ready", "t1_acc_ready", "g2_out_free"]
for k in range(12):
    v = [int(u - t0) for u in a[k] if u]
    d = np.diff(v) if len(v) > 1 else []
    print(f"{names[k]:16s} n={len(v):4d} mean_gap={np.mean(d) if len(d) else 0:7.0f}  first:", v[:30])
