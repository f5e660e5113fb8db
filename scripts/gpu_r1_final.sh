# round-1 final measurement (32-byte gather vectors): GPU tests, smoke, C3 bench (default contract line),
# reference arm, C5 bench, C3 launch list + ncu --set full of the C3 aggregation kernels, C5 launch list +
# ncu --set full of the C5 selective kernels
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 1500 python -m pytest tests/ -m gpu -q --durations=10 > gpurun_out/f_pytest.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/f_c3.json 2> gpurun_out/f_c3.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/f_ref.json 2> gpurun_out/f_ref.err
TH=$(python -c "import json;print(json.load(open('gpurun_out/f_c3.json'))['config']['theta'])")
B3="python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --eager --theta $TH"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f_c3_launches.csv $B3 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)|tc_engine" -s 0 -c 8 -o gpurun_out/f_c3_full $B3 > gpurun_out/f_ncu_c3.log 2>&1
timeout 1500 python bench.py --workload pl32m --steps 10 --warmup 3 > gpurun_out/f_c5.json 2> gpurun_out/f_c5.err
B5="python bench.py --workload pl32m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.0564"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f_c5_launches.csv $B5 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)" -s 0 -c 4 -o gpurun_out/f_c5_sparse $B5 > gpurun_out/f_ncu_c5.log 2>&1
