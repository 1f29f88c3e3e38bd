import sys, time, torch, os
sys.path.insert(0, '.')
import paper_conf_ipps_cuissf17_b200 as pp, synth
n=512
A0=torch.empty((n,n,n),dtype=torch.float64,pin_memory=True); synth.fill(A0,"random",seed=2017,nx=n,ny=n)
dA=A0.cuda(); dN=torch.empty_like(dA); torch.cuda.synchronize()
c0=1/6
r=pp.Region(0); r.map("to",dA,-1,3); r.map("from",dN); r.pipeline(0,1)
for _ in range(4):
    t=time.perf_counter(); r.launch(1,n-1,"stencil7",c0=c0,c1=c0/6); print("launch wall ms", (time.perf_counter()-t)*1e3, flush=True)
import ctypes
rt=ctypes.CDLL("libcudart.so"); fr=ctypes.c_size_t(); tot=ctypes.c_size_t()
for _ in range(3):
    t=time.perf_counter(); rt.cudaMemGetInfo(ctypes.byref(fr),ctypes.byref(tot)); print("cudaMemGetInfo ms",(time.perf_counter()-t)*1e3)
