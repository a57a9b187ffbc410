timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_gcn.py -q -x -k "hub_tiles" > gpurun_out/pytest_tiles.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/pytest_tiles.log
timeout 300 python tools/exp_tiles.py reddit 128,48,16,256 dense,150,200,400,800 2>&1 | tail -5 > gpurun_out/exp_lean.log
RDM_TILE_DBG=1 timeout 300 python tools/exp_tiles.py reddit 128,48,16 200 2>&1 | tail -1 >> gpurun_out/exp_lean.log
RDM_TILE_R=0 timeout 300 python tools/exp_tiles.py reddit 48,16 200 2>&1 | tail -1 >> gpurun_out/exp_lean.log
cat gpurun_out/exp_lean.log
