#!/bin/bash
# fp32 LAP4096: one NVTX-attributed full capture per format (summary made here) + the
# features kernel's pipe utilisation (original kernel)
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/f32 /tmp/f32
timeout 900 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o /tmp/f32/full_lap4096_f32 python tools/prof_formats.py lap4096 f32 > /dev/null 2>&1
echo "full $?"
python tools/ncu_summary.py full /tmp/f32/full_lap4096_f32.ncu-rep gpurun_out/f32/full_lap4096_f32.md > /dev/null 2>&1
for k in k_coo k_csr_rows k_ell k_merge_rows k_csr5 k_features; do
  python tools/ncu_hot.py /tmp/f32/full_lap4096_f32.ncu-rep "^$k\$" --top 15 > gpurun_out/f32/hot_$k.txt 2>/dev/null
  ncu -i /tmp/f32/full_lap4096_f32.ncu-rep --page details --csv -k regex:"^$k\$" 2>/dev/null | grep -i '"Duration\|Issue Slots Busy\|Executed Ipc Active\|DRAM Throughput\|No Eligible\|highest-utilized\|Achieved Occupancy\|Registers Per' | awk -F'","' '{print $(NF-2)" | "$(NF-1)" | "$NF}' | cut -c1-220 > gpurun_out/f32/det_$k.txt
done
ls gpurun_out/f32
