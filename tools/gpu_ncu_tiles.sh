timeout 600 ncu --set full --import-source on --clock-control none -k regex:hub_tile_kernel -c 2 -o gpurun_out/tiles_full python tools/exp_tiles.py reddit 16,128 200 > gpurun_out/ncu_tiles.log 2>&1; echo rc=$?
tail -3 gpurun_out/ncu_tiles.log
