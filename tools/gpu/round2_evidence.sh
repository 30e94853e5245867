#!/bin/bash
# round-2 evidence (summaries made on the box; the .ncu-rep files stay there):
# launch list, NVTX-attributed full captures (LAP4096, R-MAT24, R-MAT27 with A30 hot
# columns), L2/LTS throughput of the gather probe and the formats, hot-spot SASS
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/ev /tmp/ev
export NCU_TRAFFIC_JSON=gpurun_out/ev/ncu_traffic.json
cp profiles/ncu_traffic.json $NCU_TRAFFIC_JSON
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev/launches_lap4096.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --no-extra --no-variants > /dev/null 2>&1
echo "launches $?"
for cfg in lap4096 rmat24 rmat27; do
  F=""; [ $cfg == rmat27 ] && F="csr,merge,csr5"
  timeout 1500 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o /tmp/ev/full_$cfg python tools/prof_formats.py $cfg f64 $F > /dev/null 2>&1
  echo "full $cfg $?"
  python tools/ncu_summary.py full /tmp/ev/full_$cfg.ncu-rep gpurun_out/ev/full_${cfg}_f64.md --traffic $cfg f64 > /dev/null 2>&1
  for k in k_features k_csr5 k_merge_persist k_coo k_csr_vector k_csr_rows k_merge_rows k_ell; do
    python tools/ncu_hot.py /tmp/ev/full_$cfg.ncu-rep "^$k\$" --top 15 > gpurun_out/ev/hot_${cfg}_$k.txt 2>/dev/null
  done
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors.sum,lts__t_sectors.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/ev/lts_probe_rmat24.csv -k regex:k_probe -c 2 python tools/gather_probe.py rmat24 --reps 1 --modes 1 --formats none > /dev/null 2>&1
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/ev/lts_probe_rmat27.csv -k regex:k_probe -c 2 python tools/gather_probe.py rmat27 --reps 1 --modes 1 --formats none > /dev/null 2>&1
timeout 900 ncu --metrics $M --nvtx --profile-from-start off --clock-control none --csv --log-file gpurun_out/ev/lts_formats_rmat24.csv python tools/prof_formats.py rmat24 f64 > /dev/null 2>&1
timeout 900 ncu --metrics $M --nvtx --profile-from-start off --clock-control none --csv --log-file gpurun_out/ev/lts_formats_rmat27.csv python tools/prof_formats.py rmat27 f64 csr,merge,csr5 > /dev/null 2>&1
timeout 600 python tools/gather_probe.py lap4096 rmat24 rmat27 --reps 20 --modes 0,1 --formats none --out gpurun_out/ev/gather_probe.jsonl > /dev/null 2>&1
du -sh gpurun_out; ls gpurun_out/ev | wc -l
