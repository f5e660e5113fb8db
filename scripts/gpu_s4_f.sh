# session 4, call F: full-mode producer prefetch + separate bits barrier: full-mode parity tests, C3 default and
# bf16x1 lines, ncu --set full of the full-mode engine
set -x
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "aggregation_parity or integer_exact or long_accumulation or closed_forms or fused or epoch_parity or rmat or gemms or knobs or calibrate" > gpurun_out/s4f_pytest.log 2>&1
timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/s4f_c3.json 2> gpurun_out/s4f_c3.err
timeout 900 python bench.py --no-cpu-baseline --no-e2e --dense bf16x1 > gpurun_out/s4f_c3_bf1.json 2> gpurun_out/s4f_c3_bf1.err
TH=$(python -c "import json;print(json.load(open('gpurun_out/s4f_c3.json'))['config']['theta'])")
TC=$(python -c "import json;print(json.load(open('gpurun_out/s4f_c3.json'))['config']['theta_c'])")
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"tc_engine" -s 0 -c 4 -o gpurun_out/s4f_tc python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta $TH --theta-c $TC > gpurun_out/s4f_ncu.log 2>&1
PCGCN_TC_DYN_ORDER=size timeout 900 python bench.py --no-cpu-baseline --no-e2e --theta $TH --theta-c $TC > gpurun_out/s4f_c3_dynsize.json 2> /dev/null
timeout 900 python bench.py --no-cpu-baseline --no-e2e --theta $TH --theta-c $TC > gpurun_out/s4f_c3_fixed.json 2> /dev/null
PCGCN_TC_DYN_ORDER=size timeout 900 python bench.py --no-cpu-baseline --no-e2e --theta $TH --theta-c $TC > gpurun_out/s4f_c3_dynsize2.json 2> /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "multirow or partial_warp or long_rows" > gpurun_out/s4f_pytest2.log 2>&1
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
B5="python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0583 --order id"
timeout 1500 $B5 > gpurun_out/s4f_c5_mrowsort.json 2> gpurun_out/s4f_c5.err
PCGCN_SPARSE_MROW=0 timeout 900 $B5 > gpurun_out/s4f_c5_nomrow.json 2> /dev/null
timeout 900 $B5 > gpurun_out/s4f_c5_mrowsort2.json 2> /dev/null
