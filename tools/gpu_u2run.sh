cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "bf16 or smoke or guard or slot" 2>&1 | tail -3
for wl in cnn3 cnn3s cnn4; do python tools/exp_kernel_variants.py --workload $wl --precision bf16_tc --variants tree; done
