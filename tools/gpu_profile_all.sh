# Full evidence pass for profiles/: launch list, one ncu --set full per kernel, bench line, clocks.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
B="python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches.csv $B > /dev/null 2>&1
for k in me_fsbm sme_refine int_subpel_kernel; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 -o gpurun_out/prof_$k -f $B > /dev/null 2>&1
done
python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
ls gpurun_out
