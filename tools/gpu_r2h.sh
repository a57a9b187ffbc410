# round 2, call h: GPU tests (bf16 row->col wire, int8x2 fast tiles, short-row kernel);
# short-row threshold sweep on Reddit / products / papers (one rank of 8); Reddit bench
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2h_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2h_pytest.txt
timeout 600 python tools/exp_short.py reddit 128,41,16 > gpurun_out/r2h_short_reddit.txt 2>&1
timeout 900 python tools/exp_short.py products 256,100,47,32 > gpurun_out/r2h_short_products.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r2h_bench.json 2> gpurun_out/r2h_bench.err
timeout 1500 python tools/exp_short.py papers 16 8 > gpurun_out/r2h_short_papers.txt 2>&1
echo done
