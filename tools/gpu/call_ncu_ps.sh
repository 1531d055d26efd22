set -x
for v in "" "ISP_TMA_STATIC=1"; do
  tag=$([ -z "$v" ] && echo pers || echo static)
  env $v timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_p?staged -s 3 -c 1 -o gpurun_out/ps_$tag python tools/prof_one.py --variant tma --mode clamp --launches 4 > gpurun_out/ncu_$tag.log 2>&1
  tail -3 gpurun_out/ncu_$tag.log
done
ISP_P_NWC=16 ISP_P_CTAS=2 ISP_P_RING_KB=90 timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_pstaged -s 3 -c 1 -o gpurun_out/ps_pers16 python tools/prof_one.py --variant tma --mode clamp --launches 4 > gpurun_out/ncu_pers16.log 2>&1
ls -la gpurun_out
