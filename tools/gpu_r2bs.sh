# round 2, call bs: hub-tile selection threshold re-swept with the final kernels (Reddit-shaped, w = 128 / 41)
mkdir -p gpurun_out
timeout 1200 python tools/exp_tiles.py reddit 128,41 auto,250,320,500,650 > gpurun_out/r2bs_tiles_thr.txt 2>&1
echo done
