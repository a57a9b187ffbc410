# round 2, call at: end-of-session evidence — full GPU suite, bench lines (Reddit with cpu_baseline, products,
# saint, papers emulation), reference arm, launch list, ncu --set full of the SpMM kernels
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2at_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2at_pytest.txt
timeout 900 python bench.py > gpurun_out/r2at_bench.json 2> gpurun_out/r2at_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2at_products.json 2>> gpurun_out/r2at_bench.err
timeout 900 python bench.py --saint --no-cpu-baseline > gpurun_out/r2at_saint.json 2>> gpurun_out/r2at_bench.err
timeout 1500 python bench.py --emulate 8 --steps 3 --warmup 3 > gpurun_out/r2at_papers.json 2>> gpurun_out/r2at_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2at_reddit_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2at_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|hub_tile_i8|gemm_tc" -c 12 -o gpurun_out/r2at_full python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2at_ncu_full.log 2>&1
echo done
