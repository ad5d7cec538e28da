#!/bin/bash
# 3xFP16 (TG_FP32_TC): GPU tests of the path, memcheck of a small fused-U3 case, bench lines
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "fp32_tc or tc_ or smoke" > gpurun_out/pytest_h3.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_h3.log
timeout 300 compute-sanitizer --tool memcheck python -c "
import numpy as np, synth, oracle
from paper_conf_ipps_sundaramrc09_b200 import tg
for n5 in (20, 60, 120):
    img=synth.images_np(3,2,92,100); prm=synth.cnn_params_np(3,n5,92,100)
    h5,w5=synth.cnn_dims(92,100)[4]; out=np.zeros((2,9,h5,w5),np.float32)
    g,_=tg.cnn_graph(img,n5,prm,out=out); g.set(torch_runtime=True, precision=tg.TG_FP32_TC); g.plan().execute()
    ref=oracle.cnn(img,n5,prm); print('n5', n5, 'err', np.abs(out-ref).max()/np.abs(ref).max())
" > gpurun_out/sanitizer_h3.log 2>&1; echo "memcheck rc=$?"; tail -5 gpurun_out/sanitizer_h3.log
for t in cnn3s cnn3; do
  timeout 400 python bench.py --template $t --precision fp32_tc --no-cpu --per-template none > gpurun_out/bench_${t}_fp32_tc_new.json 2> /dev/null; echo "bench $t rc=$?"
  python - $t <<'PY'
import json,sys
j=json.loads(open(f"gpurun_out/bench_{sys.argv[1]}_fp32_tc_new.json").read().strip().splitlines()[-1])
print(sys.argv[1], round(j["value"]), round(j["e2e"]["value"]), {k[:7]: round(v["ms"],4) for k,v in j["roofline"]["units"].items()})
PY
done
