#!/bin/bash
# e2e of the batch CNN against the chunk size (images per chunk) and the pipeline depth
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
run() {  # $1 precision, $2 depth, $3 images per chunk cap
  px=$(( $3 * 307200 ))
  timeout 300 python bench.py --template cnn3 --precision $1 --no-cpu --depth $2 --max-chunk-px $px --steps 8 > gpurun_out/chunk_$1_$2_$3.log 2>&1
  python - "$1" "$2" "$3" <<'PY'
import json,sys
j=json.loads(open(f"gpurun_out/chunk_{sys.argv[1]}_{sys.argv[2]}_{sys.argv[3]}.log").read().strip().splitlines()[-1])
e=j["e2e"]; print(sys.argv[1:], e["chunks"], round(e["value"]), round(e["host_link"]["roofline_frac"],3), round(e["overlap"],3), round(e["host_link"]["peak_bidir_each_gbs"],1))
PY
}
for d in 3 2; do for b in 11 16 22 32; do run bf16_tc $d $b; done; done
run fp32_tc 3 11; run fp32_tc 2 16; run fp32_tc 2 22
