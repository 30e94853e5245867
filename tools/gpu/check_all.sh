nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
(time python -m pytest tests -m gpu -x -q 2>&1 | tail -15) > gpurun_out/pytest_gpu.log 2>&1
python bench.py > gpurun_out/bench.log 2>&1
python bench.py --config rmat24 --no-cpu > gpurun_out/bench_rmat24.log 2>&1
python bench.py --config rmat24 --dtype f32 --no-cpu --no-e2e > gpurun_out/bench_rmat24_f32.log 2>&1
python bench.py --dtype f32 --no-cpu --no-e2e > gpurun_out/bench_f32.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -c 3000 gpurun_out/bench.log
python tools/gather_probe.py lap4096 rmat24 --out gpurun_out/gather_probe.jsonl > gpurun_out/gather_probe.log 2>&1
tail -20 gpurun_out/gather_probe.log
