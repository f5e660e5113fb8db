B="timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.028"
PCGCN_SPARSE_MINB=1 $B > gpurun_out/t22_minb1.json 2>/dev/null
PCGCN_SPARSE_MINB=4 $B > gpurun_out/t22_minb4.json 2>/dev/null
PCGCN_SPARSE_MINB=3 $B > gpurun_out/t22_minb3.json 2>/dev/null
PCGCN_SPLIT_BYTES=0 $B > gpurun_out/t22_split.json 2>/dev/null
PCGCN_SPLIT_BYTES=0 PCGCN_SPARSE_MINB=4 $B > gpurun_out/t22_split4.json 2>/dev/null
PCGCN_SPARSE_GV=16,2 $B > gpurun_out/t22_gv162.json 2>/dev/null
PCGCN_SPARSE_GV=8,4 $B > gpurun_out/t22_gv84.json 2>/dev/null
