cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for B in 11 8 6 4 3; do
  px=$((B*307200))
  timeout 300 python bench.py --template cnn3 --precision bf16_tc --no-cpu --max-chunk-px $px --steps 5 > gpurun_out/chunk_$B.log 2>&1
  python - "$B" <<'PY'
import json,sys
j=json.loads(open(f"gpurun_out/chunk_{sys.argv[1]}.log").read().strip().splitlines()[-1])
e=j["e2e"]; print(sys.argv[1], e["chunks"], round(e["value"]), round(e["host_link"]["roofline_frac"],3), round(e["overlap"],3))
PY
done
for B in 11 6 4; do
  px=$((B*307200))
  timeout 300 python bench.py --template cnn3 --precision fp32_tc --no-cpu --max-chunk-px $px --steps 5 > gpurun_out/chunkt_$B.log 2>&1
  python - "$B" <<'PY'
import json,sys
j=json.loads(open(f"gpurun_out/chunkt_{sys.argv[1]}.log").read().strip().splitlines()[-1])
e=j["e2e"]; print("fp32_tc", sys.argv[1], e["chunks"], round(j["value"]), round(e["value"]), round(e["host_link"]["roofline_frac"],3), round(e["overlap"],3))
PY
done
