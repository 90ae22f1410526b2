cd $GRAFT_REPO_ROOT
for cfg in "0 0" "1 0" "1 6" "1 7" "1 5" "0 6"; do set -- $cfg
  python bench.py --steps 40 --warmup 3 --no-e2e --no-cpu-baseline --pipeline $1 --me-ctas $2 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('pipeline=$1 me_ctas=$2', round(d['value'],1), 'fps', round(d['ms_per_step'],3), 'ms', {k:(round(v,3) if isinstance(v,float) else v) for k,v in d['kernels_ms'].items() if k!='note'})"
done
