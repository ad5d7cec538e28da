#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for p in bf16_tc fp32; do for t in cnn3 cnn3s cnn4; do
  timeout 900 python bench.py --template $t --precision $p --no-cpu > gpurun_out/bench_${t}_$p.log 2>&1; echo "bench $t $p rc=$?"
  python - "$t" "$p" <<'PY'
import json,sys
l=json.loads(open(f"gpurun_out/bench_{sys.argv[1]}_{sys.argv[2]}.log").read().strip().splitlines()[-1])
r=l["roofline"]; e=l["e2e"]
print(f"  value {l['value']:.0f} Mpx/s  ms/step {l['ms_per_step']:.3f}  e2e {e['value']:.0f} Mpx/s  dominant {r['kernel']} {r['achieved']:.1f} TF frac {r['frac']:.2f}  units {r['units_ms_per_step']}  link {e.get('host_link',{}).get('roofline_frac')}")
PY
done; done
