# C3 theta sweep (Table III view on the Reddit-shaped graph) + ncu --set full of the C5 GEMM kernels
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 1200 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --sweep 2,0.08,0.056,0.04,0.028,0.02,0.01,0 > gpurun_out/s3p_c3_sweep.json 2> gpurun_out/s3p_c3_sweep.err
B5="python bench.py --workload pl32m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.0693"
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:"tc_engine|softmax|split_transpose" -s 0 -c 8 -o gpurun_out/s3p_c5_gemm $B5 > gpurun_out/s3p_ncu_c5g.log 2>&1
