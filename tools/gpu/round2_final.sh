#!/bin/bash
# round-2 final evidence on the final kernels: GPU parity suite, the driver's bench
# commands (ours + reference arm), then tools/gpu/round2_evidence.sh (launch list,
# NVTX-attributed full captures, LTS / gather probe) and the sanitizers
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/fin
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/fin/pytest_gpu.log 2>&1
echo "pytest $?"; tail -2 gpurun_out/fin/pytest_gpu.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/fin/bench.json 2> gpurun_out/fin/bench.err
echo "bench $?"
timeout 900 python bench.py --impl reference --gpus 1 --steps 3 --warmup 3 > gpurun_out/fin/bench_ref.json 2> gpurun_out/fin/bench_ref.err
echo "bench ref $?"
timeout 900 python bench.py --config rmat27 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/fin/bench_rmat27.json 2> gpurun_out/fin/bench_rmat27.err
echo "bench rmat27 $?"
timeout 600 python tools/feat_time.py lap4096 rmat24 > gpurun_out/fin/feat.jsonl 2>&1
bash tools/gpu/round2_evidence.sh > gpurun_out/fin/evidence.log 2>&1
echo "evidence $?"
bash tools/gpu/sanitize.sh > gpurun_out/fin/sanitize.log 2>&1
echo "sanitize $?"
du -sh gpurun_out
