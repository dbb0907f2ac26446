import sys; sys.path.insert(0,'.')
import numpy as np, torch
import paper_conf_asplos_hagedornfccgg23_b200 as fm
from oracle import attention_fp64
from workloads import FmhaConfig, make_fmha_inputs
dev=torch.device('cuda:0')
for (b,h,sq,skv,dt,mask) in [(1,1,128,128,'bf16',0),(1,2,256,256,'bf16',0),(2,3,200,520,'fp16',0),(2,3,512,512,'bf16',2),(2,3,384,384,'bf16',0),(2,2,300,77,'bf16',1)]:
    cfg=FmhaConfig('c',11,b,h,sq,skv,128,dt,mask)
    q,k,v,kl=make_fmha_inputs(cfg)
    if mask==1: kl=np.array([skv, skv//3-1][:b],dtype=np.int32)
    kld=None if kl is None else torch.from_numpy(kl).to(dev)
    o=fm.fmha_fwd(q.to(dev),k.to(dev),v.to(dev),kv_len=kld,causal=mask==2,scale=cfg.scale); torch.cuda.synchronize()
    ref=attention_fp64(q,k,v,cfg.scale,kl,causal=mask==2)
    g=o.double().cpu().numpy(); print(b,h,sq,skv,dt,mask,'maxerr',np.abs(g-ref).max(),'rel',np.linalg.norm(g-ref)/np.linalg.norm(ref), flush=True)
