# round 2, call bo: short-row SpMM entries in flight per row (U = 1 / 2 / 4)
mkdir -p gpurun_out
timeout 900 python tools/exp_short_u.py > gpurun_out/r2bo_short_u.txt 2>&1
echo done
