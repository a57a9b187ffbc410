# round 2, call bl: compute-sanitizer (memcheck / racecheck / synccheck) on small invocations incl. the round-2 kernels
mkdir -p gpurun_out
for t in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $t --print-limit 50 python tools/sanitize_small.py > gpurun_out/r2bl_sanitize_$t.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bl_sanitize_$t.txt
done
echo done
