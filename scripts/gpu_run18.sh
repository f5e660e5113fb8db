timeout 90 python tests/debug_dense.py > gpurun_out/pair_debug.log 2>&1
for u in 1 2 4; do PCGCN_PAIR_U=$u timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.028 --sweep 0.02,0.014 > gpurun_out/pairu$u.json 2> gpurun_out/pairu$u.err; done
