# N = 4 and 8 ranks time-sliced on ONE GPU over gloo: the bench's PeerStream path end to end at the
# scaling run's rank counts (functional check: not a scaling number), plus the adaptive re-split
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
for n in 4 8; do
  FEVES_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2954$n bench.py --gpus $n --steps 6 --warmup 3 --e2e-steps 3 > gpurun_out/multirank$n.json 2> gpurun_out/multirank$n.err
  echo "n=$n rc=$?"; tail -2 gpurun_out/multirank$n.err; python -c "import json; d=json.load(open('gpurun_out/multirank$n.json')); print(d['value'], d['n_gpus'], d['config']['parallelism'], [ (r['rows'], round(r['stripe_ms_mean'],3)) for r in d['per_rank']])"
done
FEVES_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29561 bench.py --gpus 4 --steps 6 --warmup 3 --e2e-steps 3 --adaptive > gpurun_out/multirank4a.json 2> gpurun_out/multirank4a.err
echo "adaptive rc=$?"; tail -2 gpurun_out/multirank4a.err
