# round 2, call bn: configuration sweep of the products-shaped 3-layer model (64 IDs) with the final kernels
mkdir -p gpurun_out
timeout 2400 python bench.py --workload products --sweep --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bn_sweep_products.json 2> gpurun_out/r2bn.err
echo done
