# Usage: bash tools/gpu_profile2.sh <tag>
TAG=${1:-r1z}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_launch_stdout.log 2>&1; echo ncu1 rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:spmm_kernel -s 8 -c 2 \
   -o gpurun_out/${TAG}_spmm python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_spmm_stdout.log 2>&1; echo ncu2 rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:gemm_tc -s 10 -c 10 \
   -o gpurun_out/${TAG}_gemm python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_gemm_stdout.log 2>&1; echo ncu3 rc=$?
