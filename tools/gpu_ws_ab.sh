# warp-specialised ME A/B: parity on the S = 64 GPU tests, then the bench line with ME_OPT_ME_WS 0 / 1
# (FLAGS: extra nvcc -D knobs, e.g. "-DFEVES_WS_CW=2")
cd $GRAFT_REPO_ROOT
for flags in ${FLAGSETS:-""}; do
  f="${flags//,/ }"
  echo "#### flags: $f"
  FEVES_NVCC_EXTRA="$f" python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
  [ -n "$TESTK" ] && timeout 900 python -m pytest tests -x -q -m gpu -k "$TESTK" 2>&1 | tail -2
  for w in ${WS:-0 1}; do
    echo "== me_ws $w"
    timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --me-ws $w 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels_ms']; print(round(d['value'],1), round(d['ms_per_step'],4), 'me', round(k['me'],4), 'sme', round(k['sme'],4), 'frac', round(d['roofline']['frac'],4))"
  done
done
