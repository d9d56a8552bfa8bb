#!/bin/bash
# Same-session comparison of environment settings (C4 two-step path):
#   tools/ab_env.sh rounds "VAR=a" "VAR=b" ...
# ms per launch of the volume / boundary / shell kernels, and their sum per double step.
N=$1; shift
AB_ARGS=${AB_ARGS:---warmup 10}
for i in $(seq 1 $N); do
  for envs in "$@"; do
    env $envs timeout 180 python tools/profile_run.py --steps 20 ${AB_ARGS} 2>&1 | tail -1 | python -c "
import sys, ast
l = sys.stdin.read(); d = ast.literal_eval(l.split(' ', 2)[2])
nv = max(1, d['volume_launches'])
vol = d['volume_ms'] / nv; bnd = d['boundary_ms'] / max(1, d['boundary_launches'])
sh = d['shell_ms'] / max(1, d['shell_launches']); oth = d['other_ms'] / nv
tot = (d['volume_ms'] + d['boundary_ms'] + d['shell_ms'] + d['other_ms']) / nv
print('$envs', 'vol %.3f' % vol, 'bnd %.4f' % bnd, 'shell %.4f' % sh, 'other %.4f' % oth, 'sum/launch %.4f' % tot)"
  done
done
