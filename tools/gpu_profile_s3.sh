# Usage: bash tools/gpu_profile_s3.sh <tag>   (launch lists + ncu --set full of the top kernels)
TAG=${1:-s3}
for W in reddit products; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/${TAG}_${W}_launches.csv python bench.py --workload $W --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_${W}_ncu_launch_stdout.log 2>&1; echo ncu-launch $W rc=$?
done
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|hub_tile" -s 12 -c 6 \
   -o gpurun_out/${TAG}_products_spmm python bench.py --workload products --steps 1 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_products_stdout.log 2>&1; echo ncu-products rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"spmm_kernel|hub_tile" -s 8 -c 8 \
   -o gpurun_out/${TAG}_reddit_spmm python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_reddit_stdout.log 2>&1; echo ncu-reddit rc=$?
