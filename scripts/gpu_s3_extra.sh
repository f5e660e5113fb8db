# SURVEY §8(f) evidence: Table III replica (RMAT series), F2 (l-layer / hidden sweep), F3 (bf16 full mode
# accuracy delta), C4 theta sweep
set -x
export PCGCN_GRAPH_CACHE=/tmp/pcgcn_graphs
timeout 1500 python bench.py --table3 --steps 20 --warmup 5 > gpurun_out/s3x_table3.json 2> gpurun_out/s3x_table3.err
timeout 1200 python bench.py --f2 "2,4,6:64,128,256" --steps 10 --warmup 3 --theta 0.05 > gpurun_out/s3x_f2.json 2> gpurun_out/s3x_f2.err
timeout 900 python bench.py --workload pubmed --f3 200 --theta 0.02 > gpurun_out/s3x_f3_pubmed.json 2> gpurun_out/s3x_f3_pubmed.err
timeout 1500 python bench.py --workload reddit --f3 100 --theta 0.05 > gpurun_out/s3x_f3_reddit.json 2> gpurun_out/s3x_f3_reddit.err
timeout 2400 python bench.py --workload sbm4m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --sweep 2,0.03,0.02,0.01,0.005 > gpurun_out/s3x_c4.json 2> gpurun_out/s3x_c4.err
