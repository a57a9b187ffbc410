# round 2, call ba: end-of-session evidence — full GPU suite, smoke, bench lines (Reddit default incl. cpu_baseline,
# products, saint, papers emulation, reference arm), launch lists, per-call SpMM DRAM traffic (both workloads),
# ncu --set full of the top kernels
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2ba_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ba_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2ba_smoke.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ba_smoke.txt
timeout 900 python bench.py > gpurun_out/r2ba_bench.json 2> gpurun_out/r2ba_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2ba_products.json 2>> gpurun_out/r2ba_bench.err
timeout 900 python bench.py --saint --no-cpu-baseline > gpurun_out/r2ba_saint.json 2>> gpurun_out/r2ba_bench.err
timeout 1500 python bench.py --emulate 8 --steps 3 --warmup 3 > gpurun_out/r2ba_papers.json 2>> gpurun_out/r2ba_bench.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r2ba_reference.json 2>> gpurun_out/r2ba_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2ba_reddit_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2ba_products_launches.csv python bench.py --workload products --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"spmm_short_kernel|spmm_kernel|hub_tile_i8|tile_colmax|tile_panels_i8|spmm_heavy" -c 24 --csv --log-file gpurun_out/r2ba_reddit_spmm_dram.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 1200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"spmm_short_kernel|spmm_kernel|hub_tile_i8|tile_colmax|tile_panels_i8|spmm_heavy" -c 36 --csv --log-file gpurun_out/r2ba_products_spmm_dram.csv python bench.py --workload products --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|hub_tile_i8|gemm_tc|spmm_short" -c 14 -o gpurun_out/r2ba_full python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2ba_ncu_full.log 2>&1
echo done
