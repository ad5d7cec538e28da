cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "3 0" "4 3379200" "5 3379200" "6 3379200" "4 0"; do
  set -- $cfg
  mc=""; [ "$2" != "0" ] && mc="--max-chunk-px $2"
  timeout 300 python bench.py --template cnn3 --precision fp32_tc --depth $1 $mc --per-template none --no-cpu --no-verify --steps 30 --warmup 3 2>/dev/null | tail -1 > /tmp/o.json
  python -c "
import json; j=json.load(open('/tmp/o.json')); e=j['e2e']
print('depth $1 mc $2', round(e['value']), 'chunks', e['chunks'], 'srf', round(e['streamed_roofline']['frac'],3), 'arena', e['arena_bytes']>>20, 'MiB')"
done
