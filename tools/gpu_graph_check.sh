#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --template edge256 --per-template cnn3:bf16_tc,cnn3s:bf16_tc --steps 20 --warmup 5 --no-cpu > gpurun_out/bench_small.json 2> gpurun_out/bench_small.err; echo "bench rc=$?"; tail -3 gpurun_out/bench_small.err
