for v in minb3 default minb5 minb6; do echo $v; if [ $v = default ]; then unset RDM_LIB_VARIANT; else export RDM_LIB_VARIANT=$v; fi; timeout 300 python tools/exp_tiles.py reddit 128,48,16,256 csr,400,800 2>&1 | tail -3; done > gpurun_out/exp_minb.log
unset RDM_LIB_VARIANT
cat gpurun_out/exp_minb.log
