# round 2, call ax: short-row SpMM kernel on an auxiliary stream beside the long-row kernel
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_ops.py -x -q -k "spmm" > gpurun_out/r2ax_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ax_pytest.txt
timeout 900 python tools/exp_conc.py > gpurun_out/r2ax_conc.txt 2>&1
for c in 0 1; do RDM_SPMM_CONC=$c timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r2ax_bench_c$c.json 2>> gpurun_out/r2ax.err; done
echo done
