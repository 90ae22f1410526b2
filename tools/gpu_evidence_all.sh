# full round evidence: tools/gpu_evidence.sh + GPU test log + stripe probe + reference arm
cd $GRAFT_REPO_ROOT
bash tools/gpu_evidence.sh > gpurun_out/evidence.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python tools/stripe_probe.py 1 2 4 8 > gpurun_out/stripe_probe.txt 2>&1
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
ls gpurun_out
