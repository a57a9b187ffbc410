set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_tiles.log 2>&1; echo bench rc=$?
tail -1 gpurun_out/bench_tiles.log | cut -c1-600
timeout 900 python tools/exp_tiles.py products 256,100,48 csr,dense,auto,800,1600 > gpurun_out/exp_tiles_products.log 2>&1; echo exp rc=$?
cat gpurun_out/exp_tiles_products.log
