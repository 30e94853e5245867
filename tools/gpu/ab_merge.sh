python -m pytest tests -m gpu -x -q -k "csr or merge" 2>&1 | tail -3
for cfg in lap4096 rmat24; do for dt in f64 f32; do
  echo "== $cfg $dt pipe"; python tools/exp.py $cfg merge csr --dtype $dt --reps 100
  echo "== $cfg $dt persist / noflat"; SPMV_CSR_FLAT=0 SPMV_MERGE_VARIANT=1 python tools/exp.py $cfg merge csr --dtype $dt --reps 100
done; done
ncu --set full --clock-control none --import-source on -k regex:'k_(csr_vector|merge_pipe|merge_persist)' -c 2 -o gpurun_out/ncu_csr_merge python tools/exp.py lap4096 csr merge --reps 1 > /dev/null 2>&1
SPMV_CSR_FLAT=0 SPMV_MERGE_VARIANT=1 ncu --set full --clock-control none --import-source on -k regex:'k_(csr_vector|merge_pipe|merge_persist)' -c 2 -o gpurun_out/ncu_csr_merge_old python tools/exp.py lap4096 csr merge --reps 1 > /dev/null 2>&1
ls gpurun_out
