# SME build-knob sweep: SME parity tests + tools/sme_probe.py (L2 flushed, events) per flag set
cd $GRAFT_REPO_ROOT
for flags in ${FLAGSETS:-""}; do
  f="${flags//,/ }"
  echo "#### flags: $f"
  FEVES_NVCC_EXTRA="$f" python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
  [ -n "$TESTK" ] && timeout 900 python -m pytest tests -x -q -m gpu -k "$TESTK" 2>&1 | tail -2
  FEVES_NVCC_EXTRA="$f" timeout 600 python tools/sme_probe.py ${CFG:-} 2>&1 | grep "sme_kernel=0" | tail -1
done
