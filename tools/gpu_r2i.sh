# round 2, call i: fast-variant loss error by tile form and wire (diagnostic)
set -x
mkdir -p gpurun_out
for a in 1 0; do for b in 1 0; do
  if [ "$a" = 1 ]; then export RDM_TILE_PIECES_FAST=1; else unset RDM_TILE_PIECES_FAST; fi
  export RDM_BF16_WIRE=$b
  timeout 300 python tools/diag_fast_loss.py >> gpurun_out/r2i_fast_loss.txt 2>&1
done; done
echo done
