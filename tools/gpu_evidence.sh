#!/bin/bash
# Round evidence in one gpurun call: GPU tests, smoke, every bench line, ncu launch lists of the
# default (edge) bench and the CNN bf16 bench, full captures of K1 and the CNN units (both precisions).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
bash tools/gpu_bench_all.sh
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"edge|cnn" --csv --log-file gpurun_out/launches_edge.csv python bench.py --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1; echo "ncu list edge rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"cnn" --csv --log-file gpurun_out/launches_cnn3_bf16.csv python bench.py --template cnn3 --precision bf16_tc --steps 2 --warmup 3 --no-cpu > /dev/null 2>&1; echo "ncu list cnn rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:edge -s 1 -c 1 -o gpurun_out/k1_full -f python tools/prof_k1.py 15 > /dev/null 2>&1; echo "k1 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_bf16_full -f python tools/prof_cnn.py 120 bf16 > /dev/null 2>&1; echo "cnn bf16 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_fp32_full -f python tools/prof_cnn.py 120 > /dev/null 2>&1; echo "cnn fp32 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_fp32tc_full -f python tools/prof_cnn.py 120 fp32tc > /dev/null 2>&1; echo "cnn fp32tc rc=$?"
