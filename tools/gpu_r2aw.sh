# round 2, call aw: GraphSAINT step A/B on one box after the pair threshold + clock-sampler start-up fix
mkdir -p gpurun_out
for i in 1 2; do
for cfg in default pair0 tps1; do
  case $cfg in pair0) export RDM_PAIR=0;; tps1) export RDM_TILE_TPS=1;; esac
  timeout 600 python bench.py --saint --no-cpu-baseline > gpurun_out/r2aw_saint_$cfg.$i.json 2>> gpurun_out/r2aw.err
  unset RDM_PAIR RDM_TILE_TPS
done; done
echo done
