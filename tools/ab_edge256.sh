#!/bin/bash
# A/B of the configs[0] line between two prebuilt trees under _exp/ (alternating runs)
cd $GRAFT_REPO_ROOT
for r in 1 2 3; do
  for v in "$@"; do
    (cd _exp/$v && timeout 300 python bench.py --template edge256 --steps 20 --warmup 5 --no-cpu --no-verify --per-template none 2>/dev/null | tail -1) > /tmp/ab.json
    python -c "
import json; j=json.load(open('/tmp/ab.json')); print('$v', 'dev_us %.2f' % (j['ms_per_step']*1e3), 'e2e_us %.2f' % (j['e2e']['ms_per_step']*1e3), 'kern_us %.2f' % (j['roofline']['kernel_ms_per_launch']*1e3))"
  done
done
