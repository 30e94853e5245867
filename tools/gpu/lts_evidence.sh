#!/bin/bash
# R-MAT ceiling evidence: the gather probe and the formats' kernels under ncu L2 (LTS) /
# L1 / DRAM throughput metrics (one replay per kernel), R-MAT 24 and R-MAT 27
python -c "import __graft_entry__ as g; g.build()" || exit 1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors.sum,lts__t_sectors.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
timeout 900 python tools/gather_probe.py rmat24 rmat27 --reps 20 --formats csr,merge,csr5 --out gpurun_out/gather_probe.jsonl > gpurun_out/gather_probe.log 2>&1
tail -12 gpurun_out/gather_probe.log
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/lts_probe_rmat24.csv -k regex:k_probe -c 4 python tools/gather_probe.py rmat24 --reps 1 --formats none > /dev/null 2>&1
timeout 900 ncu --metrics $M --nvtx --profile-from-start off --clock-control none --csv --log-file gpurun_out/lts_formats_rmat24.csv python tools/prof_formats.py rmat24 f64 > /dev/null 2>&1
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/lts_probe_rmat27.csv -k regex:k_probe -c 4 python tools/gather_probe.py rmat27 --reps 1 --formats none > /dev/null 2>&1
timeout 900 ncu --metrics $M --nvtx --profile-from-start off --clock-control none --csv --log-file gpurun_out/lts_formats_rmat27.csv python tools/prof_formats.py rmat27 f64 csr,merge,csr5 > /dev/null 2>&1
ls -la gpurun_out/*.csv
