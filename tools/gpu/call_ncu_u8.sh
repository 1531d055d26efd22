timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_fused -s 1 -c 1 -o gpurun_out/u8_fused python tools/prof_one.py --op fused3 --mode mirror --launches 3 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_stencil -s 2 -c 1 -o gpurun_out/u8_lap python tools/prof_one.py --op laplace --variant warp --mode mirror --launches 3 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_stencil -s 2 -c 1 -o gpurun_out/u8_har python tools/prof_one.py --op harris --variant warp --mode mirror --launches 3 > /dev/null 2>&1
ls gpurun_out | grep u8_
