# round 2, call an: hub tiles, 2 tiles per stage with merged bits copies — tests, kernel times, epoch
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_fast.py -x -q > gpurun_out/r2an_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2an_pytest.txt
timeout 900 ncu --metrics gpu__time_duration.sum,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:hub_tile_i8 --csv --log-file gpurun_out/r2an_tile.csv python tools/exp_tile_dbg.py 0,7,6 > gpurun_out/r2an_tile.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r2an_bench.json 2>> gpurun_out/r2an.err
echo done
