# ncu --set full of the ME kernel at BASELINE configs 1-2 (integer ME only)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
for c in ${CFGS:-1080p_sa32 cif}; do
  ncu --set full --clock-control none --import-source on -k regex:me_fsbm -s 3 -c 1 -o gpurun_out/prof_me_$c -f \
    python bench.py --config $c --steps 4 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_me_$c.log 2>&1
  python tools/ncu_summary.py gpurun_out/prof_me_$c.ncu-rep > gpurun_out/sum_me_$c.txt 2>&1
done
