# GEMM diagnosis: normal / skip converter (RDM_TC_DBG=1) / skip MMA (=2) / both (=3), fp32 and fast
for P in fp32 fast; do
for D in 0 1 2 3; do
  echo "== prec $P dbg $D"
  RDM_TC_DBG=$D RDM_PREC=$P timeout 300 python tools/time_gemm.py 2>&1 | grep -v "^core" | head -20
done; done
