# stream-structure A/B: graph per frame, plain enqueue, per-RF pipeline, SME(t) || ME(t+1) overlap (hi / lo priority)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
run() { timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline $@ 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), round(d['ms_per_step'],4), 'e2e', round(d['e2e']['value'],1) if isinstance(d.get('e2e'),dict) else None)"; }
for a in "--graph 1" "--graph 0" "--graph 0 --overlap 1"; do echo "== $a"; run $a; done
echo "== --graph 0 --overlap 1 (FEVES_OV_LO)"; FEVES_OV_LO=1 run --graph 0 --overlap 1
