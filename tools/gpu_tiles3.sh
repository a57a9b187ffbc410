timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_gcn.py -q -x -k "hub_tiles or hub_core" > gpurun_out/pytest_tiles.log 2>&1; echo pytest rc=$?
tail -5 gpurun_out/pytest_tiles.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/tiles_launches3.csv python tools/exp_tiles.py reddit 128,48,16 200,400 > gpurun_out/exp_tiles_ncu.log 2>&1; echo ncu rc=$?
timeout 600 python tools/exp_tiles.py reddit 128,48,16,256 dense,150,200,300,400,800 > gpurun_out/exp_tiles3.log 2>&1; echo exp rc=$?
cat gpurun_out/exp_tiles3.log | tail -20
