timeout 600 python -m pytest tests/test_gpu_ops.py -q -x -k "hub_tiles" > gpurun_out/pytest_tiles.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/pytest_tiles.log
timeout 300 python tools/exp_tiles.py reddit 128,48,16,256 dense,200,400,800 2>&1 | tail -4 > gpurun_out/exp_rot.log
RDM_TILE_DBG=1 timeout 300 python tools/exp_tiles.py reddit 128,48,16 200 2>&1 | tail -1 >> gpurun_out/exp_rot.log
cat gpurun_out/exp_rot.log
