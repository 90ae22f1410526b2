# SME kernel variant sweep: each tools/smehb_*.so timed by bench.py (PARITY=1: GPU tests too)
cd $GRAFT_REPO_ROOT
for f in tools/smehb_*.so; do
  FEVES_LIB=$PWD/$f python bench.py --steps 40 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$f', round(d['kernels_ms']['sme']*1000,1), 'us sme', round(d['value'],1), 'fps')"
done
if [ -n "$PARITY" ]; then
  for f in tools/smehb_*.so; do
    echo "parity $f: $(FEVES_LIB=$PWD/$f timeout 600 python -m pytest tests -x -q -m gpu 2>&1 | tail -1)"
  done
fi
