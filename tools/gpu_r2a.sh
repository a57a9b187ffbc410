set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2a_smi.txt
lscpu > gpurun_out/r2a_lscpu.txt; free -g >> gpurun_out/r2a_lscpu.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r2a_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2a_pytest.txt
timeout 600 python bench.py > gpurun_out/r2a_bench.json 2> gpurun_out/r2a_bench.err
timeout 600 tools/gather_bench > gpurun_out/r2a_gather.jsonl 2> gpurun_out/r2a_gather.err
timeout 900 ncu --set full --clock-control none -k regex:"spmm_kernel|hub_tile_kernel" -c 6 -o gpurun_out/r2a_products_spmm python bench.py --workload products --steps 1 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2a_ncu_products.log 2>&1
timeout 400 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r2a_ref.json 2> gpurun_out/r2a_ref.err
timeout 900 python bench.py --impl reference --threads 1 --steps 1 > gpurun_out/r2a_ref_1t.json 2> gpurun_out/r2a_ref_1t.err
echo done
