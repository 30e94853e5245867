# round-end evidence: GPU parity suite, bench lines, ncu launch list + full captures
set -x
python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/pytest_gpu.log
python bench.py > gpurun_out/bench_lap4096.log 2>&1
python bench.py --config rmat24 --no-cpu > gpurun_out/bench_rmat24.log 2>&1
python bench.py --dtype f32 --no-cpu --no-e2e > gpurun_out/bench_lap4096_f32.log 2>&1
python bench.py --config rmat24 --dtype f32 --no-cpu --no-e2e > gpurun_out/bench_rmat24_f32.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_lap4096.csv \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k 'regex:^k_(coo|ell|csr_vector|merge_persist|csr5|fixup)$' -c 8 \
    -o gpurun_out/full_lap4096 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k 'regex:^k_(coo|ell|csr_vector|csr_chunks|merge_persist|csr5|fixup)$' -c 12 \
    -o gpurun_out/full_rmat24 python bench.py --config rmat24 --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
python tools/gather_probe.py lap4096 rmat24 --out gpurun_out/gather_probe.jsonl > /dev/null 2>&1
ls -la gpurun_out
