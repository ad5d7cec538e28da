#!/bin/bash
# CNN iteration: GPU tests of the CNN path, cnn3/cnn4 benches (no CPU leg), ncu full captures of
# the CNN units in both precisions (tools/prof_cnn.py).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "${PYTEST_K:-cnn}" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
for t in ${TEMPLATES:-cnn3 cnn4}; do for p in ${PRECS:-fp32 bf16_tc}; do
  timeout 600 python bench.py --template $t --precision $p --no-cpu > gpurun_out/bench_${t}_$p.json 2> gpurun_out/bench_${t}_$p.log
  python -c "import json; d=json.loads(open('gpurun_out/bench_${t}_$p.json').read().strip().splitlines()[-1]); print('$t $p value', round(d['value']), 'e2e', round(d['e2e']['value']), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['roofline'].get('units_ms_per_step',{}).items()})"
done; done
if [ -n "$NCU" ]; then
  for p in $NCU; do
    arg=""; [ $p = bf16 ] && arg=bf16
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_${p}_full -f python tools/prof_cnn.py 120 $arg > gpurun_out/ncu_cnn_$p.log 2>&1; echo "ncu $p rc=$?"
  done
fi
