# round 2, call q: products-shaped epoch launch list and ncu of its GEMMs
set -x
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 200 -c 60 --csv --log-file gpurun_out/r2q_products_launches.csv python bench.py --workload products --steps 2 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2q_ncu1.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"gemm_tc_kernel" -c 9 -o gpurun_out/r2q_products_gemm python bench.py --workload products --steps 1 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2q_ncu2.log 2>&1
echo done
