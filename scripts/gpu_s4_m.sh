# session 4, call M: calibration curve with the final engine; C4 line
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 1500 python bench.py --calib-curve 41,128 > gpurun_out/s4m_calib.json 2> gpurun_out/s4m_calib.err
timeout 1500 python bench.py --workload sbm4m --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/s4m_c4.json 2> gpurun_out/s4m_c4.err
