# round 2, call bm: configuration sweep (all 16 IDs, Reddit-shaped) with the final kernels; trial pick
mkdir -p gpurun_out
timeout 1200 python bench.py --sweep --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bm_sweep.json 2> gpurun_out/r2bm.err
timeout 600 python bench.py --config trial --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bm_trial.json 2>> gpurun_out/r2bm.err
echo done
