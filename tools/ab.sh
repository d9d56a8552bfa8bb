#!/bin/bash
# Same-session A/B of two library builds on the C4 two-step path (volume / boundary / shell ms per launch).
# usage: tools/ab.sh <libA> <libB> [rounds]
A=$1; B=$2; N=${3:-3}
for i in $(seq 1 $N); do
  for lib in $A $B; do
    RAFD_LIB=$lib timeout 120 python tools/profile_run.py --warmup 10 --steps 20 2>&1 | tail -1 | python -c "
import sys, ast
l = sys.stdin.read(); d = ast.literal_eval(l.split(' ', 2)[2])
print('$(basename $lib)', 'vol %.3f' % (d['volume_ms']/d['volume_launches']), 'bnd %.4f' % (d['boundary_ms']/d['boundary_launches']), 'shell %.4f' % (d['shell_ms']/max(1,d['shell_launches'])))"
  done
done
