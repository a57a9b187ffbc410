timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_gcn.py -q -x -k "hub_tiles" > gpurun_out/pytest_tiles.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/pytest_tiles.log
timeout 300 python tools/exp_tiles.py reddit 128,48,16,256 200,400,800 2>&1 | tail -3 > gpurun_out/exp_rings.log
cat gpurun_out/exp_rings.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/tiles_launches11.csv python tools/exp_tiles.py reddit 128,48,16 400 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/tiles_launches11.csv | grep -v "at::" | sort -k3 | uniq -c -f2 
