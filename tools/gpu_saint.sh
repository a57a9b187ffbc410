set -x
timeout 900 python -m pytest tests/test_gpu_saint.py -x -q > gpurun_out/pytest_saint.log 2>&1; echo pytest rc=$?
tail -30 gpurun_out/pytest_saint.log
timeout 600 python tools/time_saint.py 1 2 4 > gpurun_out/saint_time.log 2>&1; echo time rc=$?
tail -20 gpurun_out/saint_time.log
