#!/bin/bash
# e2e vs pipeline depth (tg_set_chunking) for the link-bound lines
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for t in cnn3:fp32_tc cnn26:fp32_tc cnn3:bf16_tc edge:fp32; do
  for d in 2 3 4 5; do
    timeout 300 python bench.py --template ${t%%:*} --precision ${t##*:} --depth $d --per-template none --no-cpu --no-verify --steps 20 --warmup 3 2>/dev/null | tail -1 > gpurun_out/ds.json
    python -c "
import json; j=json.load(open('gpurun_out/ds.json')); e=j['e2e']
print('$t depth $d', round(e['value']), 'chunks', e['chunks'], 'srf', round(e['streamed_roofline']['frac'],3), 'ov', round(e['overlap'],3))"
  done
done
