# row-pipelined selective pass + xtg one-wave slices + l-layer model: parity, C3/C5 bench, Table III, F2, C5 ncu
set -x
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_pipe.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.04 > gpurun_out/pipe_c3.json 2>/dev/null
timeout 1800 python bench.py --workload pl32m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.0657 > gpurun_out/pipe_c5.json 2> gpurun_out/pipe_c5.err
timeout 1200 python bench.py --table3 --steps 20 --warmup 5 > gpurun_out/table3.json 2> gpurun_out/table3.err
timeout 1200 python bench.py --f2 "2,4,6:64,128,256" --steps 10 --warmup 3 --theta 0.04 > gpurun_out/f2_c3.json 2> gpurun_out/f2_c3.err
timeout 1800 ncu --set full --clock-control none -k regex:"sparse_(row|seg)" -s 0 -c 4 -o gpurun_out/c5_sp2 python bench.py --workload pl32m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --eager --theta 0.0657 > gpurun_out/ncu_c5b.log 2>&1
