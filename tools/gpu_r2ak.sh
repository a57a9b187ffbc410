# round 2, call ak: hub tiles with half the panel bytes per SM (RDM_TILE_DBG=8), as a CTA pair would load
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:hub_tile_i8 --csv --log-file gpurun_out/r2ak_tile_dbg.csv python tools/exp_tile_dbg.py 0,8,9,14,15 > gpurun_out/r2ak_tile_dbg.log 2>&1
echo done
