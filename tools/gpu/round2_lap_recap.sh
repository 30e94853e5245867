#!/bin/bash
# LAP4096 evidence after the round-2 COO change: launch list of the default bench command,
# NVTX-attributed full captures fp64 / fp32, hot spots, and the bench line
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/lr /tmp/lr
export NCU_TRAFFIC_JSON=gpurun_out/lr/ncu_traffic.json
cp profiles/ncu_traffic.json $NCU_TRAFFIC_JSON
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/lr/launches_lap4096.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --no-extra --no-variants > /dev/null 2>&1
echo "launches $?"
for d in f64 f32; do
  timeout 1200 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o /tmp/lr/full_lap4096_$d python tools/prof_formats.py lap4096 $d > /dev/null 2>&1
  echo "full $d $?"
  python tools/ncu_summary.py full /tmp/lr/full_lap4096_$d.ncu-rep gpurun_out/lr/full_lap4096_$d.md --traffic lap4096 $d > /dev/null 2>&1
  for k in k_coo k_ell k_csr_rows k_merge_rows k_csr5 k_features; do
    python tools/ncu_hot.py /tmp/lr/full_lap4096_$d.ncu-rep "^$k\$" --top 15 > gpurun_out/lr/hot_lap4096_${d}_$k.txt 2>/dev/null
  done
done
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/lr/bench.json 2> gpurun_out/lr/bench.err
echo "bench $?"
