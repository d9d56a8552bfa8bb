#!/bin/bash
# Small-room knob sweep (C2a / C2b, one step per sweep): Gvox/s and per-kernel times per setting.
for c in C2b C2a; do
  for envs in "X=0" "RAFD_FUSED=1" "RAFD_VOL_DYNAMIC=1" "RAFD_VOL_DYNAMIC=0" "RAFD_ZCHUNK_MAX=8" "RAFD_ZCHUNK_MAX=16" "RAFD_ZCHUNK_MAX=32" "RAFD_BND_VARIANT=0" "RAFD_BND_VARIANT=2" "RAFD_K6=1"; do
    env $envs timeout 300 python bench.py --config $c --tb 1 --steps 200 --warmup 20 --no-cpu-baseline --no-sub-records 2>/dev/null | tail -1 | python -c "
import sys, json
d = json.loads(sys.stdin.read())
k = d['kernels']
print('$c', '$envs', d['value'], 'Gvox/s', d['ms_per_step'], 'ms/step', 'vol', k['volume_ms_per_step'], 'bnd', k['boundary_ms_per_step'])"
  done
done
