timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/saint_launches.csv python tools/prof_saint.py 3 > gpurun_out/saint_ncu.log 2>&1; echo ncu rc=$?
timeout 600 python tools/time_saint.py 1 > gpurun_out/saint_time.log 2>&1; echo time rc=$?
tail -2 gpurun_out/saint_time.log
