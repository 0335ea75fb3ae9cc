import sys, os; sys.path.insert(0,'/root/repo'); sys.path.insert(0,'/root/repo/tests')
import numpy as np, workloads as W
from oracle import oracle as O
from harness import run_gpu
for env in ("", "FOP_PACKED=0"):
    if env: os.environ[env.split('=')[0]] = env.split('=')[1]
    d=W.N3['fibonacci'](T=8,C=8); x=W.make_inputs(d)
    got,op=run_gpu(d,x); ref=O.run(d,x)['Y']
    print(env, op.selected(0))
    print(got['Y'].reshape(8,8)[:, :4].T); print(ref.reshape(8,8)[:, :4].T)
