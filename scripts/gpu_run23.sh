B="timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.028"
for i in 1 2; do
PCGCN_SPARSE_MINB=1 $B > gpurun_out/t23_minb1_$i.json 2>/dev/null
PCGCN_SPARSE_MINB=4 $B > gpurun_out/t23_minb4_$i.json 2>/dev/null
PCGCN_GATHER_HINT=1 PCGCN_SPARSE_MINB=4 $B > gpurun_out/t23_h1minb4_$i.json 2>/dev/null
done
