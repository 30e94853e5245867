#!/bin/bash
# feature kernel: parity tests, warm timing, one ncu capture per matrix (LAP4096 / R-MAT24)
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 240 python -m pytest tests/test_gpu_features.py -x -q 2>&1 | tail -4
timeout 240 python -m pytest tests/test_gpu_parity.py -x -q -k "features or canonical or conversions or int64_row_ptr" 2>&1 | tail -3
timeout 120 python tools/feat_time.py lap4096 rmat24
if [ "$1" == "ncu" ]; then
  timeout 180 ncu --set full --import-source on --clock-control none -k regex:^k_features$ -s 3 -c 1 -o gpurun_out/feat_lap python tools/feat_time.py lap4096 > gpurun_out/ncu1.log 2>&1
  timeout 180 ncu --set full --import-source on --clock-control none -k regex:^k_features$ -s 3 -c 1 -o gpurun_out/feat_rmat python tools/feat_time.py rmat24 > gpurun_out/ncu2.log 2>&1
fi
