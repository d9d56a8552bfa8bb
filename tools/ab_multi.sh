#!/bin/bash
# Same-session comparison of several library builds (C4 two-step path): tools/ab_multi.sh rounds lib...
N=$1; shift
for i in $(seq 1 $N); do
  for lib in "$@"; do
    RAFD_LIB=$lib timeout 120 python tools/profile_run.py --steps 20 2>&1 | tail -1 | python -c "
import sys, ast
l = sys.stdin.read(); d = ast.literal_eval(l.split(' ', 2)[2])
print('$(basename $lib)', 'vol %.3f' % (d['volume_ms']/d['volume_launches']), 'bnd %.4f' % (d['boundary_ms']/d['boundary_launches']), 'shell %.4f' % (d['shell_ms']/max(1,d['shell_launches'])))"
  done
done
