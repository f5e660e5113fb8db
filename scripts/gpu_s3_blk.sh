# window-blocked full-mode B: parity, then C3 A/B (PCGCN_DENSE_BLOCKED) at two thetas
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/s3b2_pytest.log 2>&1
for B in 1 0; do for TH in 0.056 0.02; do
  PCGCN_DENSE_BLOCKED=$B timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --theta $TH > gpurun_out/s3b2_B${B}_t$TH.json 2> gpurun_out/s3b2_B${B}_t$TH.err
done; done
