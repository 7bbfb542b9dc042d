"""Event timeline of CTA 0 for one tc_pair launch (experiment build):
TEMCO_VARIANT=trace TEMCO_EXTRA_FLAGS="-DTEMCO_TRACE -DTEMCO_NOSTAMP" python -m paper_conf_icpp_songljkj0024_b200.build
TEMCO_LIB=build/exp/libtemco_trace.so python scripts/pair_timeline.py <config> <pair launch index> [n events]"""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as W
from paper_conf_icpp_songljkj0024_b200 import Plan
import paper_conf_icpp_songljkj0024_b200.temco as T

cfg, li = sys.argv[1], int(sys.argv[2])
nev = int(sys.argv[3]) if len(sys.argv) > 3 else 40
m = W.build_config(cfg)
p = Plan(m)
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
p.run(x, y); torch.cuda.synchronize()
T._lib.temco_debug_pair_dbg(int(os.environ.get("PAIR_DBG", "0")))
T._lib.temco_debug_pair_ev(li, None)
p.run(x, y); torch.cuda.synchronize()
ev = (ctypes.c_longlong * (16 * 512))()
T._lib.temco_debug_pair_ev(-1, ev)
ms = np.array(p.run_profiled(x, y))
steps = [(i, s) for i, s in enumerate(p.describe()["steps"]) if s["kernel"] == "tc_pair"]
print("launch", li, "out", steps[li][1]["out"], "ms %.3f" % ms[steps[li][0]])
a = np.array(ev).reshape(16, 512)
names = ["prod stage", "iss full", "iss mma done", "iss accF commit", "iss fconv", "epi accF u0", "epi ld u0",
         "epi math u0", "epi accF u1", "epi math u1", "epi P", "epi out",
         "iss accE wait", "iss accE got", "iss pF wait", "iss fconv issued"]
t0 = a[a > 0].min()
for r in range(16):
    v = a[r][a[r] > 0] - t0
    d = np.diff(v)
    off = int(os.environ.get("EV_OFF", "0"))
    print(f"{names[r]:16s} n={len(v):4d} med.step={int(np.median(d)) if len(d) else 0:6d}: " + " ".join(str(int(z)) for z in v[off:off + nev]))
# merged, time-sorted events in a steady-state window (WIN=<cycles from the median event>)
win = int(os.environ.get("WIN", "0"))
if win:
    allev = sorted((int(t - t0), names[r]) for r in range(16) for t in a[r][a[r] > 0])
    mid = allev[len(allev) // 2][0]
    prev = None
    for t, nme in allev:
        if mid <= t < mid + win:
            print(f"  {t:8d} {t - prev if prev is not None else 0:6d}  {nme}")
            prev = t
