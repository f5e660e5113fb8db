# A/B of rows-per-ticket scheduling in the selective row pass (C3, C5); parity first
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/s3t_pytest.log 2>&1
for R in 1 0; do
  PCGCN_ROWS_PER_TICKET=$R timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --theta 0.05 > gpurun_out/s3t_c3_R$R.json 2> gpurun_out/s3t_c3_R$R.err
done
for R in 1 0; do
  PCGCN_ROWS_PER_TICKET=$R timeout 1500 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0693 > gpurun_out/s3t_c5_R$R.json 2> gpurun_out/s3t_c5_R$R.err
done
timeout 1500 python -m pytest tests/test_gpu_scale.py -x -q -k c5 > gpurun_out/s3t_pytest_c5.log 2>&1
