# build, GPU tests, one bench line (summary printed)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
timeout 600 python bench.py --steps 100 --warmup 5 --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err
python - <<'PY'
import json; d=json.load(open('gpurun_out/bench.json'))
k=d['kernels_ms']; print('fps', round(d['value'],1), 'ms', round(d['ms_per_step'],4), 'me', round(k['me'],4), 'sme', round(k['sme'],4), 'int_iso', round(k['int_isolated'],4), 'e2e', round(d['e2e']['value'],1), 'me_frac', round(d['roofline']['frac'],4), 'int_frac', round(d['roofline_int']['frac'],4), d['clocks'])
PY
