#!/bin/bash
O=gpurun_out/r02ad; mkdir -p $O
for s in 0.5 0.9; do for a in "" "--gring 9" "--gring 8" "--variant 4"; do
  echo "== s=$s $a" >> $O/sweep.log
  timeout 300 python - $s $a >> $O/sweep.log 2>&1 <<'PY'
import sys, json, torch
sys.path.insert(0,'.')
import workloads
from tests.planspec import build_gpu_plan
s=float(sys.argv[1]); extra=sys.argv[2:]
opts={}
if extra and extra[0]=='--gring': opts['gring']=int(extra[1])
if extra and extra[0]=='--variant': opts['variant']=int(extra[1])
spec=workloads.c2_spec(s,s); ins=workloads.c2_inputs(workloads.C2_ROWS,0,'cuda:0')
n=workloads.C2_ROWS
plan,ids=build_gpu_plan(spec,device=0,**opts)
node=ids['s2']; outs=[torch.empty(n,dtype=torch.int32,device='cuda:0') for _ in range(3)]
nd=torch.zeros(1,dtype=torch.int64,device='cuda:0'); inputs=[(n,ins['R'])]
for _ in range(3): plan.execute(inputs,node,outs,n,n_dev=nd)
ts=[]
for _ in range(8):
    e0,e1=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
    e0.record(); plan.execute(inputs,node,outs,n,n_dev=nd); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
print(round(sorted(ts)[4],3), 'ms', plan.explain(node).split('|')[1][:120] if '|' in plan.explain(node) else '')
PY
done; done
cat $O/sweep.log
