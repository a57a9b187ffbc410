# round 2, call g: column relabelling of DRAM-resident SpMM slices (products P=1, papers one rank of 8),
# lane-mapping variants; GPU tests (bf16 wire); Reddit launch list
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2g_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2g_pytest.txt
timeout 900 python tools/exp_relabel.py products 256,100,47,32 "auto;16,4,1;8,4,1;8,2,1;8,1,4;8,2,2" > gpurun_out/r2g_relabel_products.txt 2>&1
timeout 1500 python tools/exp_relabel.py papers 16,24 "auto;4,1,1;4,1,2;4,1,4;8,1,4;8,2,1" 8 > gpurun_out/r2g_relabel_papers.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 60 -c 40 --csv --log-file gpurun_out/r2g_reddit_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-variants --no-cpu-baseline > gpurun_out/r2g_ncu.log 2>&1
echo done
