set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q -k "not reddit" > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -30 gpurun_out/pytest_gpu.log
timeout 600 python tools/time_p2p.py reddit > gpurun_out/p2p_virtual.log 2>&1; echo p2p rc=$?
tail -20 gpurun_out/p2p_virtual.log
