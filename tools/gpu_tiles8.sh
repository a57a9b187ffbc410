for d in 0 1 4 5 8 9 13; do echo dbg=$d; RDM_TILE_DBG=$d timeout 300 python tools/exp_tiles.py reddit 128,16 200 2>&1 | tail -1; done > gpurun_out/exp_dbg2.log
cat gpurun_out/exp_dbg2.log
