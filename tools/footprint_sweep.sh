#!/bin/bash
# k_volume2 (tb 2) vs the single-step kernel (tb 1) over box rooms of growing footprint: tools/footprint_sweep.sh
for d in 1536,1024,704 2048,1536,704 1536,1024,2560 2048,1536,1280 2048,1536,2560 1024,1024,2048 3072,1024,704; do
 for tb in 2 1; do
  timeout 600 python tools/profile_run.py --config C4 --dims $d --tb $tb --warmup 4 --steps 10 2>&1 | tail -1 | python -c "
import sys, ast
l = sys.stdin.read(); d = ast.literal_eval(l.split(' ', 2)[2])
nx,ny,nz=[int(v) for v in '$d'.split(',')]
n=nx*ny*nz; tb=$tb
byt = n*(1+4*4) if tb==2 else n*(1+3*4)
ms = d['volume_ms']/d['volume_launches']
print('$d', 'tb', tb, 'vol ms/launch %.3f' % ms, 'GB/s %.0f' % (byt/ms/1e6), 'bnd %.4f' % (d['boundary_ms']/d['boundary_launches']), 'shell %.4f' % (d['shell_ms']/max(1,d['shell_launches'])))" 
 done
done
