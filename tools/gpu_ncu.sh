cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
B="python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches.csv $B > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:me_fsbm -s 4 -c 1 -o gpurun_out/prof_me -f $B > gpurun_out/ncu_me.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:sme_refine -s 4 -c 1 -o gpurun_out/prof_sme -f $B > gpurun_out/ncu_sme.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:int_subpel -s 4 -c 1 -o gpurun_out/prof_int -f $B > gpurun_out/ncu_int.log 2>&1
ls -la gpurun_out
