set -x
timeout 900 python -m pytest tests/test_gpu_ablations.py tests/test_gpu_isp_bodies.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "ablation or split or tex or eq10 or peer or strips" 2>&1 | tail -3
timeout 2400 python tools/paper_sweep.py > gpurun_out/r02_paper_sweep.json 2> gpurun_out/r02_paper_sweep.err
tail -3 gpurun_out/r02_paper_sweep.err
python -c "
import json; d=json.load(open('gpurun_out/r02_paper_sweep.json'))
print(d['auto_matches_best_within_5pct']); print(json.dumps(d['geomean']))
print({m:(v['pearson_G_vs_speedup_block'], v['pearson_G_vs_speedup_auto']) for m,v in d['table3_bilateral13'].items()})
"
