# round 2, call n: ncu source-level view of the int8 tile kernels (single and paired) and the NN GEMM
set -x
mkdir -p gpurun_out
export RDM_TILE_PAIRS=0
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hub_tile_i8_kernel|gemm_tc_kernel" -c 6 -o gpurun_out/r2n_single python bench.py --steps 1 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2n_single.log 2>&1
export RDM_TILE_PAIRS=1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hub_tile_i8_pair" -c 2 -o gpurun_out/r2n_pair python bench.py --steps 1 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2n_pair.log 2>&1
echo done
