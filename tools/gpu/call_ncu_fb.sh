timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_fused_body -s 1 -c 1 -o gpurun_out/fbody2 python tools/prof_one.py --op fused3 --mode mirror --launches 3 > /dev/null 2>&1
ls gpurun_out | grep fbody
