# INT kernel variant sweep: each tools/intv_*.so timed by bench.py (INT isolated, L2 flushed)
cd $GRAFT_REPO_ROOT
for f in paper_conf_icpp_ilicmrs14_b200/libfeves_me.so tools/intv_*.so; do
  FEVES_LIB=$PWD/$f python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$f', 'int_iso_us', round(d['kernels_ms']['int_isolated']*1000,2), 'clean', round(d['kernels_ms']['int_isolated_clean_l2']*1000,2), 'fps', round(d['value'],1))"
done
if [ -n "$PARITY" ]; then
  for f in tools/intv_*.so; do
    echo "parity $f: $(FEVES_LIB=$PWD/$f timeout 600 python -m pytest tests -x -q -m gpu 2>&1 | tail -1)"
  done
fi
