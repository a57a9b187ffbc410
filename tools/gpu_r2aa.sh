# round 2, call aa: ncu --set full of the 602-wide NN GEMM, single CTA vs CTA pair
mkdir -p gpurun_out
for p in 0 1; do
RDM_PAIR=$p timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc_kernel -s 1 -c 1 -o gpurun_out/r2aa_nn_pair$p python tools/one_gemm.py > gpurun_out/r2aa_ncu$p.log 2>&1
done
echo done
