#!/bin/bash
# Build and time kernel experiment variants (-D flags) on the GPU box, then restore the normal build.
# usage: EXPS="-DU2_EXP=1 -DU2_EXP=2" TRACE_ARGS="--device" bash tools/exp_variants.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
B='import importlib.util; s=importlib.util.spec_from_file_location("b","paper_conf_ipps_sundaramrc09_b200/build.py"); b=importlib.util.module_from_spec(s); s.loader.exec_module(b); b.build()'
for e in "" $EXPS; do
  TG_NVCC_DEFS="$e" python -c "$B" > gpurun_out/exp_build.log 2>&1 || { echo "build $e failed"; tail -20 gpurun_out/exp_build.log; continue; }
  echo "== variant '$e'"
  timeout 300 python tools/trace_e2e.py $TRACE_ARGS 2>/dev/null | grep -v "^{" | awk '{print "   ", $1, $2, $3, $4, $5}'
done
python -c "$B" > /dev/null 2>&1
