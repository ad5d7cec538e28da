#!/bin/bash
# GPU tests + unit times of the CNN benches (no CPU leg): a quick check after a kernel change
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_quick.log
for t in ${TEMPLATES:-cnn3 cnn3s}; do for p in ${PRECS:-fp32 fp32_tc bf16_tc}; do
  timeout 300 python bench.py --template $t --precision $p --no-cpu --per-template none --steps 20 2>/dev/null | tail -1 > gpurun_out/q_${t}_$p.json
  python -c "
import json; j=json.load(open('gpurun_out/q_${t}_$p.json')); print('$t $p', round(j['value']), round(j['e2e']['value']), {k[:7]: round(v['ms'],4) for k,v in j['roofline']['units'].items()})"
done; done
