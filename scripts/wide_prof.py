"""MMA-issuer cycle accounting of CTA 0 for every wide-kernel group (experiment build).

TEMCO_VARIANT=trace TEMCO_EXTRA_FLAGS="-DTEMCO_TRACE -DTEMCO_NOSTAMP" python -m paper_conf_icpp_songljkj0024_b200.build
TEMCO_LIB=build/exp/libtemco_trace.so python scripts/wide_prof.py [config]
Columns: % of the issuer's cycles spent waiting for a free TMEM buffer (acc),
the epilogue's P tile (p), the output buffer (out), a full ring stage (full),
issuing MMAs (issue) -- per group, with the group's per-step time.
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
dbg = int(os.environ.get("WIDE_DBG", "0"))   # 2: epilogue does no TMEM / SMEM work
T._lib.temco_debug_wide_dbg(dbg)
p.run(x, y); torch.cuda.synchronize()
ms = np.array(p.run_profiled(x, y))
T._lib.temco_debug_wide_prof(buf)
p.run(x, y); torch.cuda.synchronize()
n = T._lib.temco_debug_wide_prof(buf)
a = np.array(buf, dtype=np.float64).reshape(64, 16)
wide = [(i, s) for i, s in enumerate(d["steps"]) if s["kernel"] == "tc_chain" and s.get("tc", {}).get("variant") == "wide"]
print(f"{n} wide launches; {len(wide)} wide steps in describe")
print("  out   ms   tiles units stages |  acc%    p%  out%  full% issue%  dec%  com%  (cycles, mma instrs, cyc/mma)")
for k, (i, s) in enumerate(wide[:n]):
    r = a[k]
    tot = r[0]
    print(f"{s['out']:5d} {ms[i]:.3f} {int(r[9]):6d} {int(r[10]):4d} {int(r[11]):4d} | " +
          " ".join(f"{100 * r[j] / tot:5.1f}" for j in (1, 2, 3, 4, 5, 7, 8)) + f"  ({int(tot)}, {int(r[6])}, {tot / max(r[6], 1):.1f})")
