# session 4, call H: full-mode pipeline shape A/B at fixed theta (chunks per stage U, stages), bf16x3 and bf16x1
set -x
TH=${TH:-0.039}; TC=${TC:-0.0663}
B3="python bench.py --no-cpu-baseline --no-e2e --steps 30 --warmup 5 --theta $TH --theta-c $TC"
for rep in 1 2; do
  timeout 600 $B3 > gpurun_out/s4h_u4_$rep.json 2> /dev/null
  PCGCN_TC_U=2 timeout 600 $B3 > gpurun_out/s4h_u2_$rep.json 2> /dev/null
  PCGCN_TC_U=1 timeout 600 $B3 > gpurun_out/s4h_u1_$rep.json 2> /dev/null
done
B1="python bench.py --no-cpu-baseline --no-e2e --steps 30 --warmup 5 --dense bf16x1 --theta 0.026 --theta-c 0.045"
timeout 600 $B1 > gpurun_out/s4h_bf1_u4.json 2> /dev/null
PCGCN_TC_U=2 timeout 600 $B1 > gpurun_out/s4h_bf1_u2.json 2> /dev/null
PCGCN_TC_U=1 timeout 600 $B1 > gpurun_out/s4h_bf1_u1.json 2> /dev/null
