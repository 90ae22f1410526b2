cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
run() { timeout 300 python bench.py --steps 60 --warmup 5 --e2e-steps 100 --no-cpu-baseline $@ 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value', round(d['value'],1), 'e2e', round(d['e2e']['value'],1))"; }
echo "== base"; run
echo "== ov hi ctas6"; run --overlap 1 --me-ctas 6
echo "== ov lo ctas6"; FEVES_OV_LO=1 run --overlap 1 --me-ctas 6
echo "== ov lo ctas7"; FEVES_OV_LO=1 run --overlap 1 --me-ctas 7
echo "== ov hi ctas7"; run --overlap 1 --me-ctas 7
echo "== no-ov ctas6"; run --me-ctas 6
