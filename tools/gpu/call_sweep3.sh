set -x
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | grep -v "^E   *\[" | tail -12 | cut -c1-200
timeout 1800 python tools/paper_sweep.py > gpurun_out/r03e_paper_sweep.json 2> gpurun_out/r03e_paper_sweep.err; tail -3 gpurun_out/r03e_paper_sweep.err
python -c "
import json; d=json.load(open('gpurun_out/r03e_paper_sweep.json')); print(d['auto_matches_best_within_5pct'], d['geomean'])"
