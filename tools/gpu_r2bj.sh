# round 2, call bj: final evidence after TN pairs — full GPU suite, smoke, bench lines, launch lists, ncu full
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2bj_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bj_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2bj_smoke.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bj_smoke.txt
timeout 900 python bench.py > gpurun_out/r2bj_bench.json 2> gpurun_out/r2bj_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2bj_products.json 2>> gpurun_out/r2bj_bench.err
timeout 900 python bench.py --saint --no-cpu-baseline > gpurun_out/r2bj_saint.json 2>> gpurun_out/r2bj_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2bj_reddit_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2bj_products_launches.csv python bench.py --workload products --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|hub_tile_i8|gemm_tc|spmm_short" -c 14 -o gpurun_out/r2bj_full python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2bj_ncu_full.log 2>&1
echo done
