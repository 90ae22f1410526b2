# build, GPU tests (TESTK filter, default all), a 100-step bench line (+ per-config lines if CFGS set)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
if [ -n "$TESTK" ]; then timeout 1200 python -m pytest tests -x -q -m gpu -k "$TESTK" 2>&1 | tail -3; else timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -3; fi
timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline > gpurun_out/tb.json 2>/dev/null
python -c "import json; d=json.load(open('gpurun_out/tb.json')); k=d['kernels_ms']; print('value', round(d['value'],1), 'ms', round(d['ms_per_step'],4), 'me', round(k['me'],4), 'sme', round(k['sme'],4), 'frac', round(d['roofline']['frac'],4), 'e2e', round(d['e2e']['value'],1))"
for c in $CFGS; do
  timeout 300 python bench.py --config $c --steps 100 --warmup 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['value'],1), 'ms', round(d['ms_per_step'],5), 'frac', round(d['roofline']['frac'],4))"
done
