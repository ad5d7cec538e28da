#!/bin/bash
# Benches of every template workload + GPU tests (one gpurun call).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
for t in edge cnn4 cnn3 cnn3s; do
  timeout 900 python bench.py --template $t $BENCH_EXTRA > gpurun_out/bench_$t.log 2>&1; echo "bench $t rc=$?"; tail -c 3000 gpurun_out/bench_$t.log; echo
done
