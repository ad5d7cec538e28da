#!/bin/bash
# ncu evidence: launch list of the default bench + full captures of K1, U2, U3.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"edge|cnn" --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu > gpurun_out/bench_ncu.log 2>&1; echo "ncu list rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:edge -s 1 -c 1 -o gpurun_out/k1_full -f python tools/prof_k1.py 15 > gpurun_out/ncu_k1.log 2>&1; echo "k1 rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_full -f python tools/prof_cnn.py 120 > gpurun_out/ncu_cnn.log 2>&1; echo "cnn rc=$?"
