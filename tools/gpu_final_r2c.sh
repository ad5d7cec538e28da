#!/bin/bash
# Round-2 closing evidence, second pass (after the U3 bias-layout change): GPU tests, smoke, the
# default bench line, the reference arm, launch lists, ncu full captures of the tensor-core CNN units
# (the FFMA kernels and K1 are unchanged since tools/gpu_final_r2b.sh), the 2-rank functional run
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -8 gpurun_out/smoke.log
t0=$(date +%s); timeout 1500 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc=$? $(( $(date +%s) - t0 )) s"
t0=$(date +%s); timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo "ref rc=$? $(( $(date +%s) - t0 )) s"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"edge" --csv --log-file gpurun_out/launches_bench_edge256.csv python bench.py --template edge256 --steps 20 --warmup 3 --no-cpu --no-verify --per-template none > /dev/null 2>&1; echo "ncu edge256 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"cnn" --csv --log-file gpurun_out/launches_bench_cnn3_bf16_tc.csv python bench.py --template cnn3 --precision bf16_tc --steps 5 --warmup 3 --no-cpu --no-verify --per-template none > /dev/null 2>&1; echo "ncu cnn3 launches rc=$?"
for pr in bf16 fp32tc; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_${pr}_full -f python tools/prof_cnn.py 120 $pr > gpurun_out/ncu_cnn_$pr.log 2>&1; echo "cnn $pr rc=$?"
done
TG_BENCH_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-verify --per-template edge256:fp32,cnn4:bf16_tc,cnn26:bf16_tc > gpurun_out/bench_2rank.json 2> gpurun_out/bench_2rank.err; echo "2rank rc=$?"
