# round 2, call br: the driver's default bench invocation on the final build + smoke
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/r2br_bench.json 2> gpurun_out/r2br_bench.err; echo "rc=$?" >> gpurun_out/r2br_bench.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2br_smoke.txt 2>&1; echo "rc=$?" >> gpurun_out/r2br_smoke.txt
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/r2br_reference.json 2>> gpurun_out/r2br_bench.err
echo done
