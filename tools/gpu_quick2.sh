#!/bin/bash
# quick check after a kernel change: selected GPU tests + unit times (tools/exp_kernel_variants.py tree)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "${PYTEST_K:-fp32_tc}" > gpurun_out/pytest_q.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_q.log
for wp in ${WPS:-cnn3:fp32_tc cnn3s:fp32_tc cnn4:fp32_tc}; do
  python tools/exp_kernel_variants.py --workload ${wp%%:*} --precision ${wp##*:} --variants tree
done
