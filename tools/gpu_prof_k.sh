# One ncu --set full capture per kernel regex in $KS (default: sme_refine), summarised in place.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
B="python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS:-}"
for k in ${KS:-sme_refine}; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s ${NCU_S:-3} -c 1 -o gpurun_out/prof_$k -f $B > gpurun_out/ncu_$k.log 2>&1
  python tools/ncu_summary.py gpurun_out/prof_$k.ncu-rep > gpurun_out/sum_$k.txt 2>&1
  python tools/sass_hist.py gpurun_out/prof_$k.ncu-rep >> gpurun_out/sum_$k.txt 2>&1
  head -60 gpurun_out/sum_$k.txt
done
