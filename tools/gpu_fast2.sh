timeout 900 python -m pytest tests/test_gpu_fast.py -x -q > gpurun_out/fast_tests.log 2>&1; echo fast-tests rc=$?
tail -3 gpurun_out/fast_tests.log
for W in reddit products; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/fast_${W}_launches.csv python bench.py --workload $W --precision fast --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-variants \
   > /dev/null 2>&1; echo ncu-launch $W rc=$?
done
for C in 8 16 32; do
  RDM_SPMM_CHUNK4=$C timeout 400 python bench.py --workload products --no-cpu-baseline --no-e2e --steps 10 > gpurun_out/chunk_$C.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/chunk_$C.json'));print('chunk4=$C', d['value'], d['phases_ms_per_step']['spmm'], d['variants'])"
done
