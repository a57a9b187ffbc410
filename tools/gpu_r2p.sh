# round 2, call p: one-rank emulations of the P = 8 shapes with per-op sampled parity
set -x
mkdir -p gpurun_out
timeout 1800 python bench.py --emulate 8 --steps 5 --warmup 3 > gpurun_out/r2p_papers_emul.json 2> gpurun_out/r2p_papers_emul.err
timeout 900 python bench.py --emulate 8 --workload products --steps 10 --warmup 3 > gpurun_out/r2p_products_emul.json 2> gpurun_out/r2p_products_emul.err
timeout 900 python bench.py --emulate 8 --workload reddit --steps 20 --warmup 3 > gpurun_out/r2p_reddit_emul.json 2> gpurun_out/r2p_reddit_emul.err
echo done
