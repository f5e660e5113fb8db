# session 4, call L: final round measurement of HEAD (stacked bf16x3 parts) — full GPU suite, smoke, default C3 line, bf16x1 line,
# C3 ncu launch list + --set full of the selective / full-mode kernels, calibration curve, C5 line
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/s4l_gpu.txt
timeout 2700 python -m pytest tests/ -m gpu -q --durations=15 > gpurun_out/s4l_pytest.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s4l_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/s4l_c3.json 2> gpurun_out/s4l_c3.err
timeout 900 python bench.py --no-cpu-baseline --no-e2e --dense bf16x1 > gpurun_out/s4l_c3_bf1.json 2> gpurun_out/s4l_c3_bf1.err
TH=$(python -c "import json;print(json.load(open('gpurun_out/s4l_c3.json'))['config']['theta'])")
TC=$(python -c "import json;print(json.load(open('gpurun_out/s4l_c3.json'))['config']['theta_c'])")
B3="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta $TH --theta-c $TC"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s4l_c3_launches.csv $B3 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"sparse_(row|seg)|tc_engine" -s 0 -c 8 -o gpurun_out/s4l_c3_full $B3 > gpurun_out/s4l_ncu_c3.log 2>&1
