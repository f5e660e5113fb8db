for gr in 8 16 32 100000; do PCGCN_TC_GROUP=$gr timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --theta 0.02 > gpurun_out/n_gr$gr.json 2>/dev/null; done
