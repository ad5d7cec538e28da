#!/bin/bash
# 3xFP16 (TG_FP32_TC): full GPU suite, memcheck of one small case, bench lines of the fp32_tc workloads
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 300 compute-sanitizer --tool memcheck python -c "
import numpy as np, synth, oracle
from paper_conf_ipps_sundaramrc09_b200 import tg
img=synth.images_np(3,2,92,100); prm=synth.cnn_params_np(3,120,92,100)
h5,w5=synth.cnn_dims(92,100)[4]; out=np.zeros((2,9,h5,w5),np.float32)
g,_=tg.cnn_graph(img,120,prm,out=out); g.set(torch_runtime=True, precision=tg.TG_FP32_TC, budget=3_000_000); p=g.plan(); p.execute()
ref=oracle.cnn(img,120,prm); print('chunks', p.json()['n_chunks'], 'err', np.abs(out-ref).max()/np.abs(ref).max())
" > gpurun_out/sanitizer_h3.log 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/sanitizer_h3.log
timeout 300 compute-sanitizer --tool racecheck python -c "
import numpy as np, synth
from paper_conf_ipps_sundaramrc09_b200 import tg
img=synth.images_np(3,1,92,100); prm=synth.cnn_params_np(3,20,92,100)
h5,w5=synth.cnn_dims(92,100)[4]; out=np.zeros((1,9,h5,w5),np.float32)
g,_=tg.cnn_graph(img,20,prm,out=out); g.set(torch_runtime=True, precision=tg.TG_FP32_TC); g.plan().execute(); print('ok')
" > gpurun_out/racecheck_h3.log 2>&1; echo "racecheck rc=$?"; tail -2 gpurun_out/racecheck_h3.log
timeout 600 python tools/micro/fp32tc_err.py > gpurun_out/fp32tc_err.log 2>&1; echo "err rc=$?"; tail -12 gpurun_out/fp32tc_err.log
for t in cnn3 cnn4 cnn3s; do
  timeout 400 python bench.py --template $t --precision fp32_tc > gpurun_out/bench_${t}_fp32_tc.json 2> gpurun_out/bench_${t}_fp32_tc.log; echo "bench $t rc=$?"
  python - $t <<'PY'
import json,sys
j=json.loads(open(f"gpurun_out/bench_{sys.argv[1]}_fp32_tc.json").read().strip().splitlines()[-1])
print(sys.argv[1], round(j["value"]), round(j["e2e"]["value"]), j["roofline"]["kernel"], j["roofline"]["bound"], round(j["roofline"]["frac"],3), j.get("cpu_baseline",{}).get("verified"))
for k,v in j["roofline"]["units"].items(): print("  ", k, round(v["ms"],4), v["flop_bound"], round(v["flop_frac"],3))
PY
done
