# round 2, call bb: 3 hub tiles per stage at narrow widths (RDM_TILE_TPS=3); 256-wide pair tiles for the 602-wide NT and products NN 100 (RDM_BN256=1)
mkdir -p gpurun_out
RDM_TILE_TPS=3 timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_fast.py -x -q > gpurun_out/r2bb_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bb_pytest.txt
for tp in 2 3; do RDM_TILE_TPS=$tp timeout 600 python tools/exp_spmm_calls.py >> gpurun_out/r2bb_calls.txt 2>&1; done
for b in 0 1; do RDM_BN256=$b timeout 300 python tools/time_gemm.py > gpurun_out/r2bb_gemm_bn256_$b.txt 2>&1; done
echo done
