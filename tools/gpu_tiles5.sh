timeout 600 python -m pytest tests/test_gpu_ops.py -q -x -k "hub_tiles" > gpurun_out/pytest_tiles.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_tiles.log
for d in 0 1 2 3; do RDM_TILE_DBG=$d timeout 300 python tools/exp_tiles.py reddit 128,48,16 200 2>&1 | tail -1; done > gpurun_out/exp_dbg.log
cat gpurun_out/exp_dbg.log
