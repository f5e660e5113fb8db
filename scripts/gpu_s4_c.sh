# session 4, call C: clean A/B at fixed theta (same box, interleaved): inline segments on/off on C3 and C5,
# multi-row on/off on C5 (degree order), segment window; C3 all-selective; bf16x1 C3 epoch parity
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
B3="python bench.py --no-cpu-baseline --no-e2e --steps 30 --warmup 5 --theta 0.04 --theta-c 0.065"
for rep in 1 2; do
  PCGCN_SEG_INLINE=1 timeout 600 $B3 > gpurun_out/s4c_c3_inl_$rep.json 2> /dev/null
  PCGCN_SEG_INLINE=0 timeout 600 $B3 > gpurun_out/s4c_c3_sep_$rep.json 2> /dev/null
done
timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 20 --warmup 5 --theta 2.0 --theta-c 2.0 > gpurun_out/s4c_c3_allsel.json 2> /dev/null
B5="python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0583"
PCGCN_SPARSE_MROW=0 timeout 1500 $B5 --order id > gpurun_out/s4c_c5_id_inl.json 2> gpurun_out/s4c_c5.err
PCGCN_SPARSE_MROW=0 PCGCN_SEG_INLINE=0 timeout 900 $B5 --order id > gpurun_out/s4c_c5_id_sep.json 2> /dev/null
PCGCN_SPARSE_MROW=0 PCGCN_SEG_AHEAD=1 timeout 900 $B5 --order id > gpurun_out/s4c_c5_id_inl_a1.json 2> /dev/null
PCGCN_SEG_INLINE=0 timeout 900 $B5 --order degree > gpurun_out/s4c_c5_deg_sep.json 2> /dev/null
PCGCN_SEG_INLINE=1 timeout 900 $B5 --order degree > gpurun_out/s4c_c5_deg_inl.json 2> /dev/null
PCGCN_SPARSE_MROW=0 timeout 1200 ncu --set full --clock-control none -k regex:"sparse_(mrow|row|seg)" -s 0 -c 4 -o gpurun_out/s4c_c5_id_sparse $B5 --order id --steps 1 --warmup 0 --eager > gpurun_out/s4c_ncu_c5.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_scale.py -m gpu -q -x -k "bf16x1" -s > gpurun_out/s4c_pytest_bf1.log 2>&1
