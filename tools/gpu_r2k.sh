# round 2, call k: full GPU tests; compute-sanitizer (memcheck / racecheck / synccheck) on small inputs;
# Reddit-shaped SpMM DRAM traffic per call (ncu --set full); default bench line
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2k_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2k_pytest.txt
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_small.py > gpurun_out/r2k_sanitize_$t.txt 2>&1; echo "rc=$?" >> gpurun_out/r2k_sanitize_$t.txt
done
timeout 900 ncu --set full --clock-control none -k regex:"spmm_short_kernel|spmm_kernel|hub_tile_i8|tile_colmax|tile_panels_i8" -c 20 -o gpurun_out/r2k_reddit_spmm python bench.py --steps 1 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2k_ncu.log 2>&1
timeout 900 python bench.py > gpurun_out/r2k_bench.json 2> gpurun_out/r2k_bench.err
echo done
