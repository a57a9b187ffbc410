# round 2, call bu: final validation after the bf16 short-row kernel — full GPU suite, smoke, default bench, products line
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2bu_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bu_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2bu_smoke.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bu_smoke.txt
timeout 900 python bench.py > gpurun_out/r2bu_bench.json 2> gpurun_out/r2bu_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2bu_products.json 2>> gpurun_out/r2bu_bench.err
timeout 900 python bench.py --saint --no-cpu-baseline > gpurun_out/r2bu_saint.json 2>> gpurun_out/r2bu_bench.err
echo done
