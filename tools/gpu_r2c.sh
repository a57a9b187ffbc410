# round 2, call c: GPU tests after the low-memory H0-column fix; SpMM lane-mapping sweep for
# narrow rows; launch list of the papers100M-shaped one-rank emulation
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2c_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2c_pytest.txt
timeout 600 python tools/exp_gvu.py reddit 41,16,128 fp32 "auto;4,3,1;8,2,2;16,1,1;16,1,2;16,1,4;8,2,1;32,1,2;4,4,1;8,4,1" > gpurun_out/r2c_gvu_reddit.txt 2>&1
timeout 900 python tools/exp_gvu.py products 256,47,32 fp32 "auto;16,4,1;32,2,1;32,2,2;16,1,4;8,2,2;8,1,4;16,1,2;4,3,1" > gpurun_out/r2c_gvu_products.txt 2>&1
timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file gpurun_out/r2c_papers_launches.csv python bench.py --emulate 8 --steps 1 --warmup 3 > gpurun_out/r2c_papers_ncu.log 2>&1
echo done
