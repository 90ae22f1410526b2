cd $GRAFT_REPO_ROOT
ncu --metrics gpu__time_duration.sum,launch__grid_size,launch__block_size,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none -c 24 --csv --log-file gpurun_out/launches_q.csv python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python - <<'PY'
import csv, collections
rows=[r for r in csv.reader(open('gpurun_out/launches_q.csv')) if len(r)>10]
h=rows[0]; d=collections.defaultdict(dict)
for r in rows[1:]:
    x=dict(zip(h,r)); d[(x['ID'],x['Kernel Name'][:40])][x['Metric Name']]=x['Metric Value']
for k,v in list(d.items())[-12:]: print(k, v)
PY
