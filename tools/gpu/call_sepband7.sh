set -x
for rep in 1 2; do
timeout 600 python tools/bench_knobs.py --cycle --env "" --env ISP_BAND_WAVES=175 --env ISP_BAND_WAVES=195 2>&1 | grep '^{'
timeout 600 python tools/bench_knobs.py --cycle --size 16384 --window 7 --env "" --env ISP_BAND_WAVES=200 --env ISP_BAND_WAVES=385 --env ISP_BAND_WAVES=400 2>&1 | grep '^{'
done
for m in clamp mirror repeat constant; do timeout 300 python tools/bench_knobs.py --mode $m --env "" 2>&1 | grep '^{'; done
