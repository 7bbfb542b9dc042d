"""CTA-0 pipeline trace of one fused-group kernel (experiment build).

TEMCO_VARIANT=trace TEMCO_EXTRA_FLAGS=-DTEMCO_TRACE python -m paper_conf_icpp_songljkj0024_b200.build
TEMCO_LIB=build/exp/libtemco_trace.so python scripts/trace_group.py [pool|chain]
Rows: 0 producer after empty-wait, 1 producer after TMA issue, 2 MMA after
full-wait, 3 MMA unit committed, 4 epilogue after acc_full, 5 epilogue unit
done, 6/7 epilogue before/after out_full, 8 MMA after acc_empty, 9/10 MMA
before/after p_full, 11 MMA out_full committed (ns from the first stamp).
"""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as W
from workloads.models import _G
from paper_conf_icpp_songljkj0024_b200 import Plan
import paper_conf_icpp_songljkj0024_b200.temco as T

which = sys.argv[1] if len(sys.argv) > 1 else "pool"
if which == "pool":   # ResNet-50 stem group: lconv 8->64, bn, relu, maxpool 3x3 s2, fconv 64->8
    g = _G("pool", 256, 112, 112, 8, "bf16", 3, rank=lambda c: 8)
    a = g.maxpool(g.relu(g.bn(g.conv(0, 64, 1, name="c0"))), 3, 2, 1)
    g.conv(a, 64, 1, name="c1")
else:                 # single-level chain at the stage-1 shape
    g = _G("chain", 256, 56, 56, 8, "bf16", 3, rank=lambda c: 8)
    a = g.relu(g.bn(g.conv(0, 64, 1, name="c0")))
    g.conv(a, 64, 1, name="c1")
m = g.m
p = Plan(m)
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
buf = (ctypes.c_longlong * (12 * 512))()
dbg = int(sys.argv[2]) if len(sys.argv) > 2 else 0
TR = hasattr(T._lib, "temco_debug_trace")   # experiment build loaded
if TR:
    T._lib.temco_debug_set(dbg)   # 1: TMA-only (MMA / epilogue idle)
for _ in range(2):
    p.run(x, y)
torch.cuda.synchronize()
if TR:
    T._lib.temco_debug_trace(buf)
print("step ms", [(s["kernel"], round(t, 3)) for s, t in zip(p.describe()["steps"], p.run_profiled(x, y))])
if not TR:
    sys.exit(0)
if os.environ.get("PROF_ONLY"):
    prof = (ctypes.c_longlong * 16)()
    T._lib.temco_debug_prof(prof)
    pv = list(prof)[:9]
    print("MMA issuer cycles: total %d  acc_empty %d  p_full %d  out_empty %d  full %d  issue %d  (mmas %d)  decode %d  commits %d" % tuple(pv))
    sys.exit(0)
T._lib.temco_debug_trace(buf)
a = np.array(buf, dtype=np.int64).reshape(12, 512)
t0 = min(v for v in a.flatten() if v)
names = ["prod_empty_ok", "prod_issued", "mma_full_ok", "mma_unit_commit", "epi_acc_ok", "epi_unit_done",
         "epi_out_wait", "epi_out_ok", "mma_accempty_ok", "mma_pfull_wait", "mma_pfull_ok", "mma_out_commit"]
for k in range(12):
    v = [int(u - t0) for u in a[k] if u]
    d = np.diff(v) if len(v) > 1 else []
    print(f"{names[k]:16s} n={len(v):4d} mean_gap={np.mean(d) if len(d) else 0:9.0f}  first:", v[:24])
prof = (ctypes.c_longlong * 16)()
T._lib.temco_debug_prof(prof)
pv = list(prof)[:9]
print("MMA issuer cycles: total %d  acc_empty %d  p_full %d  out_empty %d  full %d  issue %d  (mmas %d)  decode %d  commits %d" % tuple(pv))
