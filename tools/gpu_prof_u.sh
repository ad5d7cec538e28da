#!/bin/bash
# ncu --set full of one CNN bf16 unit (KREGEX, default u3) + source-level CSV; summary in gpurun_out.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
K=${KREGEX:-u3_tc}
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 -o gpurun_out/prof_$K -f python tools/prof_cnn.py ${N5:-120} bf16 > gpurun_out/prof_$K.log 2>&1; echo "ncu rc=$?"
ncu -i gpurun_out/prof_$K.ncu-rep --page source --csv > gpurun_out/prof_${K}_source.csv 2>/dev/null
