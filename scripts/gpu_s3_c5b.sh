# parity, C3 + C5 benches with the multi-row softmax / block tickets, ncu of all four C5 and C3 aggregations
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/s3c_pytest.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/s3c_c3.json 2> gpurun_out/s3c_c3.err
timeout 1500 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/s3c_c5.json 2> gpurun_out/s3c_c5.err
B5="python bench.py --workload pl32m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.0693"
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)" -s 0 -c 8 -o gpurun_out/s3c_c5_sparse $B5 > gpurun_out/s3c_ncu_c5.log 2>&1
B3="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.04"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)" -s 0 -c 4 -o gpurun_out/s3c_c3_sparse $B3 > gpurun_out/s3c_ncu_c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s3c_c3_launches.csv $B3 > /dev/null 2>&1
