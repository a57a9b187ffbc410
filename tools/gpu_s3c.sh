FP_R="auto;8,4,1;16,2,2;4,3,1;8,2,2;4,3,2;4,4,2"
timeout 500 python tools/exp_gvu.py reddit 128,41,16 fp32 "$FP_R" 2>&1 | tail -3
timeout 500 python tools/exp_gvu.py reddit 128,41,16 fast "auto;8,2,2;8,2,1;8,1,4;2,3,1;16,2,2;4,4,2" 2>&1 | tail -3
timeout 700 python tools/exp_gvu.py products 256,100,47 fp32 "auto;16,4,1;16,4,2;8,4,1;16,2,2;4,3,1;8,2,2;4,4,2" 2>&1 | tail -3
timeout 700 python tools/exp_gvu.py products 256,100,47 fast "auto;16,2,2;16,2,1;8,4,1;8,2,2;8,2,1;8,1,4;4,4,2" 2>&1 | tail -3
