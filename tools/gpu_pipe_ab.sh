# stream-structure A/B: graph per frame, plain enqueue, SME(t) || ME(t+1) overlap with an ME occupancy cap
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
run() { timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e $@ 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d.get('kernels_ms',{}); print(round(d['value'],1), round(d['ms_per_step'],4), 'me', k.get('me'), 'sme', k.get('sme'))"; }
for a in "--graph 1" "--graph 0 --me-ctas 6" "--graph 0 --me-ctas 7" "--graph 0 --overlap 1 --me-ctas 6" "--graph 0 --overlap 1 --me-ctas 7" "--graph 0 --overlap 1 --me-ctas 5"; do echo "== $a"; run $a; done
