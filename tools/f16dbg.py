import numpy as np, torch, sys
sys.path.insert(0,'.')
import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
from oracle import oracle as O
for (N,C,H,Wd,K) in [(1,64,8,8,128),(2,64,14,14,128),(2,72,28,28,200)]:
    l=wl.LAYERS['r50_c64_56_f16'].with_(N=N,C=C,H=H,W=Wd,K=K)
    X,dY=wl.make_inputs(l)
    p=W.plan(l.N,l.C,l.H,l.W,l.K,l.R,l.S,l.pad,'f16')
    dW=W.as_krsc(W.bfc(p,torch.from_numpy(X).cuda(),torch.from_numpy(dY).cuda())); torch.cuda.synchronize()
    got=dW.cpu().numpy(); ref=O.bfc_c(X,dY,3,3,1)
    print(p, 'err', O.rel_max_err(got,ref), 'got[0,0,0,:4]', got[0,0,0,:4], 'ref', ref[0,0,0,:4], flush=True)
