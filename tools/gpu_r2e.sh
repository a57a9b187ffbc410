# round 2, call e: int8 hub tiles (kind::i8) — GPU tests, piece-form comparison, Reddit bench
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2e_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2e_pytest.txt
timeout 900 python tools/exp_tile_pieces.py reddit 128,41,16 8,2,3 auto,200,100 > gpurun_out/r2e_pieces_reddit.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r2e_bench.json 2> gpurun_out/r2e_bench.err
timeout 900 python tools/exp_tile_pieces.py products 256,47 8,2 auto > gpurun_out/r2e_pieces_products.txt 2>&1
echo done
