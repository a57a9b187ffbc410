for V in "" cg ca; do
  export RDM_LIB_VARIANT=$V
  [ -z "$V" ] && unset RDM_LIB_VARIANT
  echo "== variant ${V:-ldg}"
  timeout 300 python tools/exp_gvu.py reddit 128,41 fp32 "auto" 2>&1 | tail -2
  timeout 300 python tools/exp_gvu.py reddit 128,41 fast "auto" 2>&1 | tail -2
  timeout 400 python tools/exp_gvu.py products 256,47 fp32 "auto" 2>&1 | tail -2
done
