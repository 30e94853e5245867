#!/bin/bash
# full GPU parity suite + default bench line (round checkpoints)
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider 2>&1 | tail -6
if [ "$1" != "nobench" ]; then
  timeout 600 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
  tail -3 gpurun_out/bench_default.err
  python -c "
import json; d=json.load(open('gpurun_out/bench_default.json'))
print('value', d['value'], 'features', d['features']['ms'], d['features']['gbs'], 'roof', d['roofline']['frac'])
for f,p in d['per_format'].items(): print(f, p.get('ms_mean'), p.get('frac_of_peak'))
"
fi
