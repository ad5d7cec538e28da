#!/bin/bash
# End-of-round evidence: tests, smoke, every bench line, ncu lists and full captures (gpu_evidence.sh),
# compute-sanitizer memcheck / racecheck / synccheck of the smoke run, the paper's Table 2 re-run.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
bash tools/gpu_evidence.sh
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 10 python __graft_entry__.py smoke > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY" gpurun_out/sanitize_$tool.log | tail -2
done
timeout 1200 python tools/paper_table2.py > gpurun_out/paper_table2_b200.jsonl 2> gpurun_out/table2.err; echo "table2 rc=$?"
