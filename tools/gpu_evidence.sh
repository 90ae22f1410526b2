# Round evidence: full bench line (defaults), launch list, one ncu --set full per kernel, per-config bench lines
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv,noheader > gpurun_out/gpu.txt
python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
B="python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --launch-skip 90 -c 60 --csv --log-file gpurun_out/launches.csv $B > /dev/null 2>&1
for k in me_fsbm sme_refine int_; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 -o gpurun_out/prof_$k -f $B > /dev/null 2>&1
done
for c in cif 1080p_sa32 1080p_sa64_4rf 2160p_sa128; do
  timeout 600 python bench.py --config $c --steps 30 --warmup 3 --cpu-budget 5 > gpurun_out/cfg_$c.json 2> gpurun_out/cfg_$c.err
done
FEVES_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 10 --warmup 3 --e2e-steps 5 > gpurun_out/multirank.json 2> gpurun_out/multirank.err
ls gpurun_out
