# round 2, call bd: products epoch with 256-wide pair tiles for the masked NT products too (RDM_BN256=1) vs default
mkdir -p gpurun_out
for i in 1 2; do for b in def 1; do
  if [ $b = 1 ]; then export RDM_BN256=1; fi
  timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bd_products_$b.$i.json 2>> gpurun_out/r2bd.err
  unset RDM_BN256
done; done
echo done
