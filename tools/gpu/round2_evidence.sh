#!/bin/bash
# round-2 evidence: sanitizers, launch list, NVTX-attributed full captures (LAP4096, R-MAT24,
# R-MAT27 with A30 hot columns), L2/LTS throughput of the gather probe and the formats
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/ev
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_workload.py > gpurun_out/ev/sanitize_$tool.log 2>&1
  echo "$tool exit $?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|sanitize workload done" gpurun_out/ev/sanitize_$tool.log | head -3
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev/launches_lap4096.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --no-extra --no-variants > /dev/null 2>&1
echo "launches $?"
timeout 900 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o gpurun_out/ev/full_lap4096_f64 python tools/prof_formats.py lap4096 f64 > /dev/null 2>&1
echo "full lap $?"
timeout 900 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o gpurun_out/ev/full_rmat24_f64 python tools/prof_formats.py rmat24 f64 > /dev/null 2>&1
echo "full rmat24 $?"
timeout 1500 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o gpurun_out/ev/full_rmat27_f64 python tools/prof_formats.py rmat27 f64 csr,merge,csr5 > /dev/null 2>&1
echo "full rmat27 $?"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors.sum,lts__t_sectors.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/ev/lts_probe_rmat24.csv -k regex:k_probe -c 2 python tools/gather_probe.py rmat24 --reps 1 --modes 1 --formats none > /dev/null 2>&1
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/ev/lts_probe_rmat27.csv -k regex:k_probe -c 2 python tools/gather_probe.py rmat27 --reps 1 --modes 1 --formats none > /dev/null 2>&1
timeout 900 ncu --metrics $M --nvtx --profile-from-start off --clock-control none --csv --log-file gpurun_out/ev/lts_formats_rmat27.csv python tools/prof_formats.py rmat27 f64 csr,merge,csr5 > /dev/null 2>&1
timeout 600 python tools/gather_probe.py lap4096 rmat24 rmat27 --reps 20 --formats none --out gpurun_out/ev/gather_probe.jsonl > /dev/null 2>&1
ls -la gpurun_out/ev
