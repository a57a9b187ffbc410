# round 2, call ae: epoch A/B of the CTA-pair GEMM policy (RDM_PAIR=0 vs auto), Reddit + products
mkdir -p gpurun_out
for i in 1 2; do
for p in 0 auto; do
  if [ $p = auto ]; then unset RDM_PAIR; else export RDM_PAIR=0; fi
  timeout 600 python bench.py --no-cpu-baseline --no-variants --no-e2e --steps 20 > gpurun_out/r2ae_reddit_$p.$i.json 2>> gpurun_out/r2ae.err
  timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-variants --no-e2e > gpurun_out/r2ae_products_$p.$i.json 2>> gpurun_out/r2ae.err
done; done
unset RDM_PAIR
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:gemm_tc -c 40 --csv --log-file gpurun_out/r2ae_reddit_gemm_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
echo done
