#!/bin/bash
# bench lines: default (LAP4096 fp64 + R-MAT24 blocks), LAP4096 fp32, R-MAT27 on one GPU
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/b
timeout 900 python bench.py > gpurun_out/b/default.json 2> gpurun_out/b/default.err; echo "default $?"
timeout 600 python bench.py --dtype f32 --no-cpu --no-extra > gpurun_out/b/lap_f32.json 2> gpurun_out/b/lap_f32.err; echo "f32 $?"
timeout 1200 python bench.py --config rmat27 --steps 20 --no-cpu --no-e2e > gpurun_out/b/rmat27.json 2> gpurun_out/b/rmat27.err; echo "rmat27 $?"
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/b/reference.json 2> gpurun_out/b/reference.err; echo "ref $?"
