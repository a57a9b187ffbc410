# round 2, call az: fused hi|lo 3xTF32 MMAs (8 instead of 12 tcgen05.mma per k-block) — parity, per-call times, trace, epoch
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_gemm_fuse.py tests/test_gpu_gemm_pair.py tests/test_gpu_ops.py -k "gemm or fuse or pair" -x -q > gpurun_out/r2az_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2az_pytest.txt
for f in 0 1; do RDM_PAIR=0 RDM_FUSE_HILO=$f timeout 300 python tools/time_gemm.py > gpurun_out/r2az_gemm_p0_f$f.txt 2>&1; done
timeout 300 python tools/time_gemm.py > gpurun_out/r2az_gemm_default.txt 2>&1
for cfg in fuse0 fuse1 pair0; do
  case $cfg in fuse0) export RDM_FUSE_HILO=0;; pair0) export RDM_PAIR=0;; esac
  timeout 600 python bench.py --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2az_bench_$cfg.json 2>> gpurun_out/r2az.err
  timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2az_products_$cfg.json 2>> gpurun_out/r2az.err
  unset RDM_FUSE_HILO RDM_PAIR
done
echo done
