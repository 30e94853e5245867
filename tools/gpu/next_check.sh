#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_features.py tests/test_gpu_hot.py -x -q > gpurun_out/nc_pytest.log 2>&1; tail -2 gpurun_out/nc_pytest.log
timeout 120 python tools/feat_time.py lap4096 rmat24
timeout 900 python tools/exp_hot.py rmat27 f64
timeout 300 python tools/exp_hot.py rmat24 f64 csr5,merge
