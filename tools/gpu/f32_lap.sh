#!/bin/bash
# LAP4096 fp32: NVTX-attributed full capture of one run per format (summary + hot spots made on the box)
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/f32 /tmp/f32
timeout 900 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o /tmp/f32/full_lap python tools/prof_formats.py lap4096 f32 > gpurun_out/f32/ncu.log 2>&1
echo "full $?"
python tools/ncu_summary.py full /tmp/f32/full_lap.ncu-rep gpurun_out/f32/full_lap4096_f32.md > gpurun_out/f32/sum.log 2>&1
for k in k_csr5 k_merge_persist k_merge_rows k_coo k_csr_vector k_csr_rows k_ell; do
  python tools/ncu_hot.py /tmp/f32/full_lap.ncu-rep "^$k\$" --top 25 > gpurun_out/f32/hot_$k.txt 2>/dev/null
  python tools/ncu_sass.py /tmp/f32/full_lap.ncu-rep "^$k\$" > gpurun_out/f32/sass_$k.txt 2>/dev/null
done
ls -la gpurun_out/f32
