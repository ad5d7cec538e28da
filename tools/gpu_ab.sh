#!/bin/bash
# Same-box A/B of kernel variants (tools/exp_kernel_variants.py, prebuilt here) + the CNN GPU parity tests.
# usage: gpu_ab.sh "<variants>" "<workload:precision ...>" [pytest selection]
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
V=$1; WL=$2; SEL=${3:-tests/test_gpu_cnn.py}
for wp in $WL; do
  timeout 900 python tools/exp_kernel_variants.py --prebuilt --workload ${wp%%:*} --precision ${wp##*:} --variants $V --steps 200
done 2>&1 | tee gpurun_out/ab.jsonl
if [ "$SEL" != "none" ]; then timeout 1500 python -m pytest $SEL -q -x 2>&1 | tail -5; fi
