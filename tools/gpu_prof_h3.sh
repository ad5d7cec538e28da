#!/bin/bash
# ncu full capture of the 3xFP16 U2/U3 (cnn3 large, fp32_tc)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"h3" -s 2 -c 2 -o gpurun_out/cnn_fp32tc_full -f python tools/prof_cnn.py 120 fp32tc > gpurun_out/ncu_cnn_fp32tc.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/ncu_cnn_fp32tc.log
