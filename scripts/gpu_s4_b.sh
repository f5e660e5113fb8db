# session 4, call B: inline long-row segments + BF16X1 on kind::f16 (one bf16 part):
# targeted GPU tests, C3 default / no-inline / bf16x1 lines, C5 degree order (inline), ncu of C5's multi-row F=32 pass
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_dist.py -m gpu -q -x -k "aggregation_parity or knobs or partial_warp or long_rows or epoch_parity or fused or peer or sharded" > gpurun_out/s4b_pytest.log 2>&1
timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/s4b_c3.json 2> gpurun_out/s4b_c3.err
PCGCN_SEG_INLINE=0 timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/s4b_c3_noinl.json 2> gpurun_out/s4b_c3_noinl.err
timeout 900 python bench.py --no-cpu-baseline --no-e2e --dense bf16x1 > gpurun_out/s4b_c3_bf1.json 2> gpurun_out/s4b_c3_bf1.err
B5="python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0583"
timeout 1500 $B5 --order degree --grain block > gpurun_out/s4b_c5_deg.json 2> gpurun_out/s4b_c5_deg.err
PCGCN_SPARSE_MROW=0 timeout 900 $B5 --order id --grain block > gpurun_out/s4b_c5_id_nomrow.json 2> gpurun_out/s4b_c5_id_nomrow.err
timeout 1200 ncu --set full --clock-control none -k regex:"sparse_(mrow|row)" -s 0 -c 3 -o gpurun_out/s4b_c5_sparse $B5 --order degree --grain block --steps 1 --warmup 0 --eager > gpurun_out/s4b_ncu_c5.log 2>&1
