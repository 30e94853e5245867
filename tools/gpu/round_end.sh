# round-end evidence in one call: parity suite, bench lines, ncu launch list + full captures
# (summarised on the box so that gpurun_out stays small), sanitizers
set -x
python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/pytest_gpu.log
python bench.py > gpurun_out/bench_lap4096.log 2>&1
python bench.py --config rmat24 --no-cpu > gpurun_out/bench_rmat24.log 2>&1
python bench.py --dtype f32 --no-cpu --no-e2e > gpurun_out/bench_lap4096_f32.log 2>&1
python bench.py --config rmat24 --dtype f32 --no-cpu --no-e2e > gpurun_out/bench_rmat24_f32.log 2>&1
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_lap4096.csv \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
mkdir -p /tmp/ncu
ncu --set full --clock-control none --import-source on -k 'regex:^k_(coo|ell|csr_vector|csr_rows|merge_persist|merge_rows|csr5|fixup)$' -c 8 \
    -o /tmp/ncu/full_lap4096 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k 'regex:^k_(coo|ell|csr_vector|csr_rows|csr_chunks|merge_persist|merge_rows|csr5|fixup)$' -c 12 \
    -o /tmp/ncu/full_rmat24 python bench.py --config rmat24 --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/launches_lap4096.csv gpurun_out/r01_launches_lap4096.md
python tools/ncu_summary.py full /tmp/ncu/full_lap4096.ncu-rep gpurun_out/r01_ncu_full_lap4096_f64.md --traffic lap4096 f64
python tools/ncu_summary.py full /tmp/ncu/full_rmat24.ncu-rep gpurun_out/r01_ncu_full_rmat24_f64.md --traffic rmat24 f64 --formats coo,csr,hyb,merge,csr5
cp profiles/ncu_traffic.json gpurun_out/ncu_traffic.json
for k in merge_rows csr_rows coo csr5; do python tools/ncu_hot.py /tmp/ncu/full_lap4096.ncu-rep $k --top 12 > gpurun_out/hot_lap4096_$k.txt 2>&1; done
python tools/gather_probe.py lap4096 rmat24 --out gpurun_out/gather_probe.jsonl > /dev/null 2>&1
du -sh gpurun_out; ls gpurun_out
