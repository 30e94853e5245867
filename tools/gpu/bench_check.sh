#!/bin/bash
# default bench line (lap4096 + R-MAT24 blocks) and a functional N=2 check on one GPU
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
echo "default rc=$?"; tail -3 gpurun_out/bench_default.err
timeout 600 python bench.py --gpus 2 --dist-backend gloo --steps 5 --warmup 3 --no-e2e > gpurun_out/bench_g2_lap.json 2> gpurun_out/bench_g2_lap.err
echo "g2 lap rc=$?"; tail -3 gpurun_out/bench_g2_lap.err
timeout 600 python bench.py --gpus 2 --dist-backend gloo --config rmat24 --steps 5 --warmup 3 > gpurun_out/bench_g2_rmat.json 2> gpurun_out/bench_g2_rmat.err
echo "g2 rmat rc=$?"; tail -3 gpurun_out/bench_g2_rmat.err
