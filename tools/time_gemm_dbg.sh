for d in 0 1 2 3; do echo "--- dbg $d"; RDM_NO_PF=1 RDM_TC_DBG=$d timeout 300 python tools/time_gemm.py 2>&1 | grep -E "NN 602|core 16384|TN 602"; done
