# Usage: bash tools/gpu_ncu_spmm.sh <tag> [kernel-regex] [count]
TAG=${1:-x}; KRE=${2:-spmm_kernel}; CNT=${3:-2}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:${KRE} -s 8 -c ${CNT} \
   -o gpurun_out/${TAG} python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e \
   > gpurun_out/${TAG}_stdout.log 2>&1; echo ncu rc=$?
