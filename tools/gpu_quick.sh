cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
timeout 600 python bench.py --steps 100 --warmup 5 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err
python - <<'PY'
import json; d=json.load(open('gpurun_out/bench.json'))
print({k: d[k] for k in ('value','ms_per_step','kernels_ms','clocks')}); print(d['roofline']['frac'], d['roofline_me_only']['frac'], d['e2e']['value'], d['roofline_int']['frac'])
PY
B="python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline"
ncu --set full --clock-control none --import-source on -k regex:${NCU_K:-me_fsbm} -s 4 -c 1 -o gpurun_out/prof_q -f $B > gpurun_out/ncu_q.log 2>&1
