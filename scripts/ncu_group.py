"""Index of a group's launch among the plan's tc_chain launches (for ncu -s):
ncu_group.py <config> <out id> [kernel substring]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W
from paper_conf_icpp_songljkj0024_b200 import Plan
cfg, out = sys.argv[1], int(sys.argv[2])
kind = sys.argv[3] if len(sys.argv) > 3 else "tc_chain"
p = Plan(W.build_config(cfg))
steps = [s for s in p.describe()["steps"] if s["kernel"].startswith(kind)]
print([i for i, s in enumerate(steps) if s["out"] == out][0])
