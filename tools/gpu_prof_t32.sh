#!/bin/bash
# ncu full capture of the 3xTF32 U2/U3 (cnn3 large, fp32_tc)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"t32" -s 2 -c 2 -o gpurun_out/cnn_t32_full -f python tools/prof_cnn.py 120 t32 > gpurun_out/ncu_cnn_t32.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/ncu_cnn_t32.log
