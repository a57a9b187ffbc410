for d in 0 1 2 3; do RDM_TILE_DBG=$d timeout 300 python tools/exp_tiles.py reddit 128,48,16 200 2>&1 | tail -1; done > gpurun_out/exp_dbg.log
cat gpurun_out/exp_dbg.log
