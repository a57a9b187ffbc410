# round 2, call am: hub tiles with 2 tiles per pipeline stage (RDM_TILE_TPS) — tests, kernel times, epoch
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_fast.py -x -q > gpurun_out/r2am_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2am_pytest.txt
for tp in 1 2; do
RDM_TILE_TPS=$tp timeout 900 ncu --metrics gpu__time_duration.sum,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:hub_tile_i8 --csv --log-file gpurun_out/r2am_tile_tp$tp.csv python tools/exp_tile_dbg.py 0,7,6 > gpurun_out/r2am_tile_tp$tp.log 2>&1
done
for tp in 1 2; do RDM_TILE_TPS=$tp timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r2am_bench_tp$tp.json 2>> gpurun_out/r2am.err; done
echo done
