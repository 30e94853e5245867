#!/bin/bash
# after the round-2 CSR batch changes: R-MAT full captures (fp64 24/27, fp32 24), LTS of the
# formats, hot spots, and the bench lines (default, R-MAT 24, R-MAT 27) on the final kernels
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/rc /tmp/rc
export NCU_TRAFFIC_JSON=gpurun_out/rc/ncu_traffic.json
cp profiles/ncu_traffic.json $NCU_TRAFFIC_JSON
for spec in "rmat24 f64" "rmat24 f32" "rmat27 f64 csr,merge,csr5"; do
  set -- $spec
  timeout 1500 ncu --set full --import-source on --nvtx --profile-from-start off --clock-control none -o /tmp/rc/full_$1_$2 python tools/prof_formats.py $1 $2 $3 > /dev/null 2>&1
  echo "full $1 $2 $?"
  python tools/ncu_summary.py full /tmp/rc/full_$1_$2.ncu-rep gpurun_out/rc/full_$1_$2.md --traffic $1 $2 > /dev/null 2>&1
  for k in k_csr_vector k_csr_chunks k_csr5 k_coo k_merge_persist; do
    python tools/ncu_hot.py /tmp/rc/full_$1_$2.ncu-rep "^$k\$" --top 15 > gpurun_out/rc/hot_$1_$2_$k.txt 2>/dev/null
  done
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors.sum,lts__t_sectors.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
timeout 900 ncu --metrics $M --nvtx --profile-from-start off --clock-control none --csv --log-file gpurun_out/rc/lts_formats_rmat24.csv python tools/prof_formats.py rmat24 f64 > /dev/null 2>&1
timeout 900 ncu --metrics $M --nvtx --profile-from-start off --clock-control none --csv --log-file gpurun_out/rc/lts_formats_rmat27.csv python tools/prof_formats.py rmat27 f64 csr,merge,csr5 > /dev/null 2>&1
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/rc/bench.json 2> gpurun_out/rc/bench.err
echo "bench $?"
timeout 900 python bench.py --config rmat24 --steps 50 --warmup 5 --no-cpu > gpurun_out/rc/bench_rmat24.json 2> gpurun_out/rc/bench_rmat24.err
echo "bench rmat24 $?"
timeout 900 python bench.py --config rmat27 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/rc/bench_rmat27.json 2> gpurun_out/rc/bench_rmat27.err
echo "bench rmat27 $?"
timeout 600 python bench.py --dtype f32 --steps 50 --warmup 5 --no-cpu --no-e2e --no-extra > gpurun_out/rc/bench_f32.json 2> gpurun_out/rc/bench_f32.err
echo "bench f32 $?"
du -sh gpurun_out/rc
