# build, (optional) GPU tests, then the ME variant sweep (tools/mev_*.so)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
[ -n "$TESTS" ] && (timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -2)
bash tools/me_variants.sh
