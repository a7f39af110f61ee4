for r in 1 2; do for it in 15 18 20 22; do HSORT_LIB=paper_conf_ipps_gowanlockk18a_b200/ab/k32_$it.so timeout 200 python tools/f32_bench.py 2>&1 | head -1; done; done > gpurun_out/r02x_k32_ab.txt
