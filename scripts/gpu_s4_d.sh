# session 4, call D: evict-first far rows (PCGCN_NEAR_ROWS) on C5; Table III with the one-part bf16 full mode
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "knobs or long_rows" > gpurun_out/s4d_pytest.log 2>&1
B5="python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0583"
for rep in 1 2; do
  PCGCN_SPARSE_MROW=0 timeout 1500 $B5 --order id > gpurun_out/s4d_c5_id_near_$rep.json 2> gpurun_out/s4d_c5.err
  PCGCN_SPARSE_MROW=0 PCGCN_NEAR_ROWS=0 timeout 900 $B5 --order id > gpurun_out/s4d_c5_id_nonear_$rep.json 2> /dev/null
done
PCGCN_SPARSE_MROW=0 PCGCN_NEAR_ROWS=8192 timeout 900 $B5 --order id > gpurun_out/s4d_c5_id_near8k.json 2> /dev/null
PCGCN_SPARSE_MROW=0 PCGCN_NEAR_ROWS=65536 timeout 900 $B5 --order id > gpurun_out/s4d_c5_id_near64k.json 2> /dev/null
timeout 900 $B5 --order degree > gpurun_out/s4d_c5_deg_near.json 2> /dev/null
PCGCN_SPARSE_MROW=0 timeout 1200 ncu --set full --clock-control none -k regex:"sparse_(mrow|row|seg)" -s 0 -c 2 -o gpurun_out/s4d_c5_id_near $B5 --order id --steps 1 --warmup 0 --eager > gpurun_out/s4d_ncu_c5.log 2>&1
timeout 1500 python bench.py --table3 --dense bf16x1 --steps 10 --warmup 3 > gpurun_out/s4d_table3_bf1_tile.json 2> gpurun_out/s4d_table3.err
timeout 1500 python bench.py --table3 --dense bf16x1 --order id --grain block --steps 10 --warmup 3 > gpurun_out/s4d_table3_bf1_block.json 2>> gpurun_out/s4d_table3.err
