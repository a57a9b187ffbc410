# End-of-session profile set: bench lines, launch lists (both precisions), ncu --set full of the top kernels.
# ncu reports are exported to CSV on the box and kept only if small (gpurun copies back <= 64 MiB).
TAG=${1:-s3f}
PART=${2:-all}
if [ "$PART" = all ] || [ "$PART" = bench ]; then
timeout 400 python bench.py > gpurun_out/${TAG}_bench_reddit.json 2> gpurun_out/${TAG}_bench_reddit.err; echo bench-reddit rc=$?
timeout 400 python bench.py --workload products --no-cpu-baseline > gpurun_out/${TAG}_bench_products.json 2>/dev/null; echo bench-products rc=$?
timeout 400 python bench.py --saint --no-cpu-baseline --no-variants > gpurun_out/${TAG}_bench_saint.json 2>/dev/null; echo bench-saint rc=$?
for P in fp32 fast; do for W in reddit products; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/${TAG}_${W}_${P}_launches.csv python bench.py --workload $W --precision $P --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-variants \
   > /dev/null 2>&1; echo ncu-launch $W $P rc=$?
done; done
fi
if [ "$PART" = all ] || [ "$PART" = ncu ]; then
for P in fp32 fast; do
R=/tmp/${TAG}_reddit_${P}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|hub_tile|gemm_tc|to_bf16|tile_panels|xent" -s 40 -c 12 \
   -o $R python bench.py --precision $P --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-variants \
   > gpurun_out/${TAG}_ncu_reddit_${P}.log 2>&1; echo ncu-full reddit $P rc=$?
ncu -i $R.ncu-rep --page raw --csv > gpurun_out/${TAG}_reddit_${P}_raw.csv 2>/dev/null
ls -la $R.ncu-rep
[ $(stat -c %s $R.ncu-rep) -lt 20000000 ] && cp $R.ncu-rep gpurun_out/
done
du -sh gpurun_out
fi
