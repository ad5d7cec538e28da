#!/bin/bash
# Round-2 check: GPU tests, the default bench line, the 2-rank (gloo, one GPU) bench run, configs[4]
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log
fi
if [ -z "$SKIP_BENCH" ]; then
  t0=$(date +%s)
  timeout 1200 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc=$? $(( $(date +%s) - t0 )) s"
  tail -3 gpurun_out/bench_default.err
fi
if [ -n "$RUN_REF" ]; then
  t0=$(date +%s)
  timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$? $(( $(date +%s) - t0 )) s"
fi
if [ -n "$RUN_2RANK" ]; then
  TG_BENCH_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-verify --per-template edge256:fp32,cnn4:bf16_tc,cnn26:bf16_tc > gpurun_out/bench_2rank.json 2> gpurun_out/bench_2rank.err; echo "2rank rc=$?"; tail -5 gpurun_out/bench_2rank.err
fi
if [ -n "$RUN_C5" ]; then
  free -g | head -2
  for pr in ${C5_PRECS:-fp32}; do
    timeout 1500 python tools/config5.py --rank 0 --world 8 --precision $pr > gpurun_out/config5_rank0of8_$pr.json 2> gpurun_out/config5_$pr.err; echo "config5 $pr rc=$?"; tail -3 gpurun_out/config5_$pr.err
  done
fi
