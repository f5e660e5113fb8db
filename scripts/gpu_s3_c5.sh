# session 3: remaining GPU tests (deep-model cap fix), C3 ncu capture of the selective gather
# (DRAM + L2->L1 bytes), C5 bench (HBM-bound showcase) and its ncu capture
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 2400 python -m pytest tests/ -m gpu -q --durations=15 > gpurun_out/s3b_pytest.log 2>&1
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.04"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)" -s 0 -c 4 -o gpurun_out/s3_c3_sparse $B > gpurun_out/s3_ncu_c3.log 2>&1
timeout 2400 python bench.py --workload pl32m --steps 10 --warmup 3 > gpurun_out/s3_c5.json 2> gpurun_out/s3_c5.err
B5="python bench.py --workload pl32m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.0657"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s3_c5_launches.csv $B5 > gpurun_out/s3_ncu_c5l.log 2>&1
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)" -s 0 -c 4 -o gpurun_out/s3_c5_sparse $B5 > gpurun_out/s3_ncu_c5.log 2>&1
