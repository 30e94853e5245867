#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 python -m pytest tests/test_gpu_matgen.py -x -q 2>&1 | tail -3
timeout 300 python -m pytest tests/test_gpu_dist.py -x -q 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_dist2.py -x -q 2>&1 | tail -30
