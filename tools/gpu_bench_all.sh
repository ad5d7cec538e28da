#!/bin/bash
# Benches of every template workload in the three CNN precisions + GPU tests (one gpurun call).
# Writes gpurun_out/bench_<template>_<precision>.json (the JSON line) and .log (stderr).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
if [ -z "$SKIP_TESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
fi
t0=$(date +%s); timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.log; echo "bench default rc=$? ($(( $(date +%s) - t0 )) s)"
for t in ${TEMPLATES:-edge cnn4 cnn3 cnn3s}; do
  for p in fp32 fp32_tc bf16_tc; do
    [ "$t" = edge ] && [ "$p" != fp32 ] && continue
    steps=5; [ "$t" != edge ] && steps=20   # CNN steps are 1-2 ms: time 20 of them
    timeout 900 python bench.py --template $t --precision $p --steps $steps $BENCH_EXTRA > gpurun_out/bench_${t}_$p.json 2> gpurun_out/bench_${t}_$p.log
    echo "bench $t $p rc=$?"
    python -c "import json,sys; d=json.loads(open('gpurun_out/bench_${t}_$p.json').read().strip().splitlines()[-1]); print(' value', round(d['value']), 'e2e', round(d['e2e']['value']), 'frac', round(d['roofline']['frac'],3), d['roofline']['kernel'], 'units', {k: round(v,3) for k,v in d['roofline'].get('units_ms_per_step',{}).items()})"
  done
done
