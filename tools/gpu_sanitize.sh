#!/bin/bash
# compute-sanitizer (memcheck, racecheck) on small runs of every kernel family.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for tool in memcheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 10 python __graft_entry__.py smoke > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY" gpurun_out/sanitize_$tool.log | tail -2
done
timeout 600 compute-sanitizer --tool memcheck --print-limit 10 python tools/micro/edge_probe.py 256 256 > gpurun_out/sanitize_tma.log 2>&1; echo "tma memcheck rc=$?"; grep "ERROR SUMMARY" gpurun_out/sanitize_tma.log
