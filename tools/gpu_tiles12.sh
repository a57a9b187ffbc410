for d in 0 1 2 3 16 17 19; do echo dbg=$d; RDM_TILE_DBG=$d timeout 120 ncu --metrics gpu__time_duration.sum --clock-control none --csv -k regex:hub_tile -c 3 python tools/exp_tiles.py reddit 16 400 2>/dev/null | grep hub_tile | tail -1 | awk -F'","' '{print $NF}'; done > gpurun_out/exp_dbg3.log 2>&1
cat gpurun_out/exp_dbg3.log
