#!/bin/bash
# Round-2 ncu evidence: launch list of the headline bench command, full captures of K1 and of
# the CNN units (bf16_tc, fp32_tc, fp32 on cnn3), summaries written into gpurun_out/
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"edge|cnn" --csv --log-file gpurun_out/launches_bench_edge.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-verify --per-template none > gpurun_out/bench_ncu.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"cnn" --csv --log-file gpurun_out/launches_bench_cnn3_bf16_tc.csv python bench.py --template cnn3 --precision bf16_tc --steps 2 --warmup 3 --no-cpu --no-verify --per-template none > gpurun_out/bench_ncu_cnn.log 2>&1; echo "ncu list cnn rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:edge -s 1 -c 1 -o gpurun_out/k1_full -f python tools/prof_k1.py 15 > gpurun_out/ncu_k1.log 2>&1; echo "k1 rc=$?"
for pr in bf16 fp32tc fp32; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_${pr}_full -f python tools/prof_cnn.py 120 $pr > gpurun_out/ncu_cnn_$pr.log 2>&1; echo "cnn $pr rc=$?"
done
