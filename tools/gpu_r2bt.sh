# round 2, call bt: bf16 short-row SpMM kernel for the fast variant — tests, per-call A/B, fast epochs
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_fast.py tests/test_gpu_bias.py tests/test_gpu_ops.py -x -q > gpurun_out/r2bt_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bt_pytest.txt
timeout 900 python tools/exp_short_bf.py > gpurun_out/r2bt_short_bf.txt 2>&1
for v in 0 1; do
  RDM_SPMM_SHORT_BF=$v timeout 600 python bench.py --precision fast --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bt_reddit_fast_$v.json 2>> gpurun_out/r2bt.err
  RDM_SPMM_SHORT_BF=$v timeout 900 python bench.py --workload products --precision fast --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bt_products_fast_$v.json 2>> gpurun_out/r2bt.err
done
echo done
