#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_edge.py tests/test_gpu_split.py -m gpu -q -x > gpurun_out/pytest_edge.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_edge.log
timeout 600 python bench.py --template edge256 --per-template none --steps 20 --warmup 5 > gpurun_out/bench_edge256.json 2> gpurun_out/bench_edge256.err; echo "bench rc=$?"; tail -3 gpurun_out/bench_edge256.err
