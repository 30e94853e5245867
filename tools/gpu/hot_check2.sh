#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_hot.py tests/test_gpu_parity.py -x -q > gpurun_out/hot_pytest.log 2>&1; tail -3 gpurun_out/hot_pytest.log
timeout 900 python bench.py --steps 50 --warmup 5 --no-extra --no-cpu --no-e2e > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python -c "
import json; d=json.load(open('gpurun_out/bench_default.json'))
print('value', d['value'], 'roof', d['roofline']['frac'])
for f,p in d['per_format'].items(): print(f, round(p.get('ms_mean'),4), round(p.get('frac_of_peak'),3))
"
timeout 300 python tools/exp_hot.py rmat24 f64 > gpurun_out/exp24.log 2>&1; tail -8 gpurun_out/exp24.log
timeout 900 python tools/exp_hot.py rmat27 f64
