for h in 1 0 1 0; do PCGCN_GATHER_HINT=$h timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.028 > gpurun_out/hintb$h.$RANDOM.json 2>/dev/null; done
