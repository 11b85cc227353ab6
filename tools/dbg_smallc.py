import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200 import torch_api as T
from synthetic import conv_inputs
import oracle
shape=(2, 3, 23, 23, 64, 7, 7, 3, 2)
for math in (mu.MATH_BF16, mu.MATH_TF32):
    d=mu.desc(*shape, math)
    x,w,dy=conv_inputs(*shape, seed=1, kind="int")
    dt=torch.bfloat16 if math==2 else torch.float32
    xd=torch.from_numpy(x).cuda().to(dt); wd=torch.from_numpy(w).cuda().to(dt)
    ws=torch.empty(8<<20, dtype=torch.uint8, device="cuda")
    print("launch", math, flush=True)
    y=T.conv_forward(mu.Handle(0), d, [(1,2)], xd, wd, workspace=ws)
    torch.cuda.synchronize()
    ref=oracle.conv_forward(x,w,3,2)
    print("maxerr", np.max(np.abs(y.double().cpu().numpy()-ref)), flush=True)
