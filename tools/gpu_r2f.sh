# round 2, call f: GPU tests with the hot-row panel; ncu of the int8 tiles + residual (Reddit);
# hot-panel experiment (products); papers100M-shaped one-rank emulation (permuted and un-permuted)
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2f_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2f_pytest.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hub_tile_i8_kernel|spmm_kernel" -c 4 -o gpurun_out/r2f_reddit_spmm python bench.py --steps 1 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2f_ncu.log 2>&1
timeout 900 python tools/exp_hot.py products 256,100,47,32 > gpurun_out/r2f_hot_products.txt 2>&1
timeout 1500 python bench.py --emulate 8 --steps 5 --warmup 3 > gpurun_out/r2f_papers_emul.json 2> gpurun_out/r2f_papers_emul.err
timeout 1500 python bench.py --emulate 8 --workload papers-local --steps 5 --warmup 3 > gpurun_out/r2f_papers_local.json 2> gpurun_out/r2f_papers_local.err
echo done
