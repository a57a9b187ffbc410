# round 2, call ap: SpMM time vs dense-operand row pitch; pair policy for single-tile short contractions (epoch)
mkdir -p gpurun_out
timeout 900 python tools/exp_ld.py > gpurun_out/r2ap_ld.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2ap_bench.json 2>> gpurun_out/r2ap.err
echo done
