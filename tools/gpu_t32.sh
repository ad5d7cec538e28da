#!/bin/bash
# 3xTF32 CNN path: GPU tests, sanitizer on one small case, and bench lines of cnn3/cnn4 fp32_tc
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "tc or t32 or fp32_tc" > gpurun_out/pytest_t32.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_t32.log
for t in cnn3 cnn4; do
  timeout 400 python bench.py --template $t --precision fp32_tc --no-cpu > gpurun_out/bench_${t}_fp32_tc.log 2>&1; echo "bench $t rc=$?"
  python - $t <<'PY'
import json,sys
j=json.loads(open(f"gpurun_out/bench_{sys.argv[1]}_fp32_tc.log").read().strip().splitlines()[-1])
print(sys.argv[1], round(j["value"]), round(j["e2e"]["value"]), j["roofline"]["kernel"], round(j["roofline"]["frac"],3))
for k,v in j["roofline"]["units"].items(): print("  ", k, round(v["ms"],4), v.get("flop_bound"), round(v["flop_frac"],3))
PY
done
