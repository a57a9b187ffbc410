# round 2, call bg: short-row threshold sweep with the up-front (col, val) kernel (64-entry batch above 32)
mkdir -p gpurun_out
timeout 900 python tools/exp_short_thr.py > gpurun_out/r2bg_thr.txt 2>&1
echo done
