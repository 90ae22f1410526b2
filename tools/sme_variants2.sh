# staged-SME variant sweep: the probe (L2 flushed, CUDA events) under several build knobs
cd $GRAFT_REPO_ROOT
for flags in "" "-DFEVES_SME2_PITCH=128" "-DFEVES_SME2_PITCH=128 -DFEVES_SME2_REGION=90000 -DFEVES_SME2_MINB=2" "-DFEVES_SME2_PITCH=64"; do
  echo "== flags: $flags"
  FEVES_NVCC_EXTRA="$flags" timeout 600 python tools/sme_probe.py 2>&1 | tail -4
done
