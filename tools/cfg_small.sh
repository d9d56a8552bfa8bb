#!/bin/bash
# Small rooms (C2a / C2b) under each single-step tile configuration (RAFD_VOL_CFG) and both
# sweep modes: Gvox/s and ms per step from bench.py (graph-timed), one line each.
for c in C2a C2b; do
  for tb in 1 2; do
    for cfg in 0 1 2 3; do
      RAFD_VOL_CFG=$cfg timeout 300 python bench.py --config $c --tb $tb --steps 200 --warmup 20 --no-cpu-baseline --no-sub-records 2>/dev/null | tail -1 | python -c "
import sys, json
d = json.loads(sys.stdin.read())
k = d['kernels']
print('$c tb=$tb cfg=$cfg', d['value'], 'Gvox/s', d['ms_per_step'], 'ms/step', 'vol', k['volume_ms_per_step'], 'bnd', k['boundary_ms_per_step'], 'shell', k['shell_ms_per_step'])"
    done
  done
done
