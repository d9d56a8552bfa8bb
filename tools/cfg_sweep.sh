#!/bin/bash
# Bench the configs with one and two steps per sweep (numbers for DESIGN.md / profiles).
for cfg in "C2a" "C2b" "C3" "C3 --precision 64" "C4"; do
  for tb in 1 2; do
    line=$(timeout 300 python bench.py --no-cpu-baseline --steps 100 --tb $tb --config $cfg 2>/dev/null)
    echo "$line" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg tb=$tb', d['value'], 'Gvox/s', d['ms_per_step'], 'ms/step vol', d['roofline']['avg_launch_ms'], 'frac', d['roofline']['frac'], 'shell/step', d['kernels']['shell_ms_per_step'], 'bnd/step', d['kernels']['boundary_ms_per_step'], 'e2e', d['e2e']['value'])" 2>&1 | tail -1
  done
done
