import sys, os, ctypes; sys.path.insert(0, os.getcwd())
import torch, numpy as np
import workloads as W
from paper_conf_icpp_songljkj0024_b200 import Plan
import paper_conf_icpp_songljkj0024_b200.temco as T
torch.zeros(1).cuda()
a = (ctypes.c_int * 5)()
print("attrs err", T._lib.temco_debug_tc_attrs(a), list(a))
m = W.resnet18_cifar(batch=3, dtype='bf16', height=16, width=16)
p = Plan(m)
x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
y = torch.empty(p.output_shape(), device="cuda")
try:
    p.run(x, y); torch.cuda.synchronize(); print("ok")
except Exception as e:
    print("ERR", e)
    print("attrs after", T._lib.temco_debug_tc_attrs(a), list(a))
