for C in 4096 8192 40000; do
  echo "== chain $C"
  [ $C = 4096 ] && (timeout 600 python -m pytest tests/test_gpu_gcn.py tests/test_gpu_ops.py -x -q -k "full_size or gemm" 2>&1 | tail -1)
  RDM_TN_CHAIN=$C timeout 400 python bench.py --workload products --no-cpu-baseline --no-e2e --no-variants > gpurun_out/ch.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/ch.json'));print(d['value'], d['phases_ms_per_step']['gemm'])"
done
