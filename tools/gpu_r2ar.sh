# round 2, call ar: residual SpMM lane mapping at w = 128 (G = 16 / 32), repeated
mkdir -p gpurun_out
for i in 1 2; do timeout 600 python tools/exp_u.py fp32 w128 >> gpurun_out/r2ar_u.txt 2>&1; done
echo done
