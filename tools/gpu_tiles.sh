set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_ops.py -q -x -k "hub_tiles or hub_core" > gpurun_out/pytest_tiles.log 2>&1; echo pytest rc=$?
tail -30 gpurun_out/pytest_tiles.log
timeout 600 python tools/exp_tiles.py reddit 128,48,16,256 > gpurun_out/exp_tiles.log 2>&1; echo exp rc=$?
cat gpurun_out/exp_tiles.log | tail -20
