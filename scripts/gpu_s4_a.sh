# session 4, call A: FADD2 + multi-row short-row layout: targeted GPU tests, C3 default / bf16x1 lines,
# C5 with the multi-row F=32 pass (id and degree order) and without it
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "aggregation_parity or knobs or partial_warp or long_rows or epoch_parity or fused" > gpurun_out/s4a_pytest.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/s4a_c3.json 2> gpurun_out/s4a_c3.err
timeout 900 python bench.py --no-cpu-baseline --no-e2e --dense bf16x1 > gpurun_out/s4a_c3_bf1.json 2> gpurun_out/s4a_c3_bf1.err
B5="python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0583"
timeout 1500 $B5 --order id --grain block > gpurun_out/s4a_c5_id.json 2> gpurun_out/s4a_c5_id.err
timeout 900 $B5 --order degree --grain block > gpurun_out/s4a_c5_deg.json 2> gpurun_out/s4a_c5_deg.err
PCGCN_SPARSE_MROW=0 timeout 900 $B5 --order degree --grain block > gpurun_out/s4a_c5_deg_nomrow.json 2> gpurun_out/s4a_c5_deg_nomrow.err
