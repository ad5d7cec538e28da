#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cnn -s 3 -c 3 -o gpurun_out/cnn_tc_full -f python tools/prof_cnn.py 120 bf16 > gpurun_out/ncu_cnn_tc.log 2>&1; echo "cnn tc rc=$?"
