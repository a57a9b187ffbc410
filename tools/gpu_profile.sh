# Usage: bash tools/gpu_profile.sh <tag>   (run under gpurun; writes gpurun_out/<tag>_*)
TAG=${1:-r1}
set -x
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo pytest rc=$?
tail -5 gpurun_out/${TAG}_pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.log 2>&1; echo bench rc=$?
tail -2 gpurun_out/${TAG}_bench.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_launch_stdout.log 2>&1; echo ncu1 rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:spmm_kernel -s 8 -c 2 \
   -o gpurun_out/${TAG}_spmm python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_spmm_stdout.log 2>&1; echo ncu2 rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:gemm -s 6 -c 3 \
   -o gpurun_out/${TAG}_gemm python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_ncu_gemm_stdout.log 2>&1; echo ncu3 rc=$?
ls -la gpurun_out/
