# round 2, call al: hub tiles — per-stage issue cost (16 = skip the bits bulk copy)
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:hub_tile_i8 --csv --log-file gpurun_out/r2al_tile_dbg.csv python tools/exp_tile_dbg.py 7,23,31,18 > gpurun_out/r2al_tile_dbg.log 2>&1
echo done
