# round 2, call j: full GPU tests; fast-variant loss diagnostic; compute-sanitizer on small inputs;
# input-specialisation controls at full size; products bench + ncu traffic; GraphSAINT x6; papers emulation
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2j_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2j_pytest.txt
timeout 300 python tools/diag_fast_loss.py > gpurun_out/r2j_fast_loss.txt 2>&1
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_small.py > gpurun_out/r2j_sanitize_$t.txt 2>&1; echo "rc=$?" >> gpurun_out/r2j_sanitize_$t.txt
done
for w in reddit-er reddit-noise reddit-row; do
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --no-variants >> gpurun_out/r2j_controls.jsonl 2>> gpurun_out/r2j_controls.err
done
timeout 1200 python bench.py --workload products --steps 10 --warmup 3 > gpurun_out/r2j_products.json 2> gpurun_out/r2j_products.err
timeout 900 ncu --set full --clock-control none -k regex:"spmm_short_kernel|spmm_kernel|hub_tile_i8" -c 9 -o gpurun_out/r2j_products_spmm python bench.py --workload products --steps 1 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2j_ncu_products.log 2>&1
for i in 1 2 3 4 5 6; do timeout 300 python bench.py --saint --steps 20 --warmup 5 --no-cpu-baseline >> gpurun_out/r2j_saint.jsonl 2>> gpurun_out/r2j_saint.err; done
timeout 1500 python bench.py --emulate 8 --steps 5 --warmup 3 > gpurun_out/r2j_papers_emul.json 2> gpurun_out/r2j_papers_emul.err
echo done
