cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
for c in cif 1080p_sa32 1080p_sa64_4rf 2160p_sa128; do
  timeout 600 python bench.py --config $c --steps 30 --warmup 3 --no-cpu-baseline > gpurun_out/cfg_$c.json 2> gpurun_out/cfg_$c.err
  python -c "import json; d=json.load(open('gpurun_out/cfg_$c.json')); print('$c', round(d['value'],1), 'fps', d['kernels_ms'], 'frac', round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value'],1))" || tail -3 gpurun_out/cfg_$c.err
done
