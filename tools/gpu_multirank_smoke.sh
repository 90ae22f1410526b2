# 2 ranks on ONE GPU over gloo: exercises bench.py's torchrun / ShardedStream path end to end
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
FEVES_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 10 --warmup 3 --e2e-steps 5 > gpurun_out/multirank.json 2> gpurun_out/multirank.err
echo rc=$?; tail -3 gpurun_out/multirank.err; cat gpurun_out/multirank.json | cut -c1-600
