#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_hot.py -x -q 2>&1 | tail -4
timeout 300 python tools/exp_hot.py rmat24 f64
timeout 300 python tools/exp_hot.py rmat24 f32
timeout 300 python tools/exp_hot.py lap4096 f64 csr,csr5,merge
timeout 900 python tools/exp_hot.py rmat27 f64
