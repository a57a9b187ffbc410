# round 2, call aq: residual SpMM nnz-in-flight (U) sweep at the Reddit-shaped widths
mkdir -p gpurun_out
timeout 900 python tools/exp_u.py > gpurun_out/r2aq_u.txt 2>&1
echo done
