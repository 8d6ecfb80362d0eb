# Model of the DRAM lines a C5 batch touches for every brick shape a0 x a1 x a2 of 32 or 64 cells (profiles/model_r02_c5_bricks.txt).
import numpy as np, synth, itertools
ext=(1024,4096,8192)
b,o=synth.config_queries("C5",nq=65536,seed=synth.CONFIGS["C5"]["seed"]+1003, extents=ext)
m=o!=synth.COUNT
b=b[m]; lo=b[:,:,0]; hi=b[:,:,1]
alg=np.prod(hi-lo+1,axis=1).sum()*4
print("alg GB", alg/1e9)
res=[]
for a0 in (1,2,4,8):
  for a1 in (1,2,4,8,16,32):
    for a2 in (1,2,4,8,16,32):
      if a0*a1*a2 not in (32,64): continue
      nb=np.ones(len(b))
      for d,a in enumerate((a0,a1,a2)):
        nb*= hi[:,d]//a - lo[:,d]//a + 1
      lines = nb*(a0*a1*a2*4/128)
      res.append((lines.sum()*128/1e9, (a0,a1,a2)))
for r in sorted(res)[:12]: print(round(r[0],2), r[1], round(r[0]/(alg/1e9),2))
print("rowmajor-ish (1,1,32):", [r for r in res if r[1]==(1,1,32)])
print("current (1,4,8):", [r for r in res if r[1]==(1,4,8)])
