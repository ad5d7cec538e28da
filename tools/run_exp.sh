V=$1; shift
for w in "$@"; do
python tools/exp_kernel_variants.py --prebuilt --workload ${w%%:*} --precision ${w##*:} --variants $V 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: j=json.loads(l); print('$w', j['variant'], {k: round(v,4) for k,v in j['unit_ms'].items()})
    except Exception: print(l.rstrip()[:200])
"
done
