# round 2, call ao: full GPU suite + Reddit / products bench lines after the 2-tiles-per-stage hub tiles
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2ao_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ao_pytest.txt
timeout 600 python bench.py > gpurun_out/r2ao_bench.json 2> gpurun_out/r2ao_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2ao_products.json 2>> gpurun_out/r2ao_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2ao_reddit_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2ao_ncu.log 2>&1
echo done
