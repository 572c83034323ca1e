import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import time, torch, numpy as np, synth
from paper_conf_micro_khorasanieas18_b200 import vpps
H=E=256; C=5
rng=np.random.default_rng(0)
shapes=vpps.param_shapes("binary",H,E,C); P=synth.init_params(shapes,rng)
m=vpps.Model("binary",H,E,C,cluster=16,dataflow=True)
params=torch.zeros(m.n_floats,device="cuda"); grads=torch.zeros_like(params)
for n,_ in shapes: m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
m.bind(params,grads)
X=torch.from_numpy(synth.input_table(rng,4096,E)).float().cuda(); dX=torch.zeros_like(X)
scripts=[m.build_script(synth.config_batch("tgt",i)) for i in range(16)]
for s in scripts: s.upload()
for i in range(20): m.fwd_bwd_sgd(scripts[i%16],X,dX,lr=1e-3,weight_decay=0.0)
torch.cuda.synchronize()
N=500
e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
t=time.perf_counter(); e0.record()
for i in range(N): m.fwd_bwd_sgd(scripts[i%16],X,dX,lr=1e-3,weight_decay=0.0)
e1.record(); th=time.perf_counter()-t
torch.cuda.synchronize(); tg=e0.elapsed_time(e1)/1e3
print(f"host enqueue {th/N*1e6:.1f} us/step, device {tg/N*1e6:.1f} us/step (no flush, back to back)")
