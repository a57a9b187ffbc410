# round 2, call bk: final evidence (xent with the label logit from registers) — full GPU suite, smoke, bench lines,
# launch lists; ncu --set full of the top kernels kept small (the gpurun_out merge limit is 64 MiB)
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2bk_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bk_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2bk_smoke.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bk_smoke.txt
timeout 900 python bench.py > gpurun_out/r2bk_bench.json 2> gpurun_out/r2bk_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2bk_products.json 2>> gpurun_out/r2bk_bench.err
timeout 900 python bench.py --saint --no-cpu-baseline > gpurun_out/r2bk_saint.json 2>> gpurun_out/r2bk_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2bk_reddit_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2bk_products_launches.csv python bench.py --workload products --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"spmm_kernel|hub_tile_i8|gemm_tc|spmm_short" -c 8 -o /tmp/r2bk_full python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2bk_ncu_full.log 2>&1
ncu -i /tmp/r2bk_full.ncu-rep --page raw --csv > gpurun_out/r2bk_full_raw.csv 2>/dev/null
du -sh gpurun_out
echo done
