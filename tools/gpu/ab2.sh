python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for dt in f64 f32; do
  echo "== lap $dt staged-flat / pipe"; python tools/exp.py lap4096 csr merge --dtype $dt --reps 200
  echo "== lap $dt unstaged-flat / persist"; SPMV_CSR_STAGE=0 SPMV_MERGE_VARIANT=1 python tools/exp.py lap4096 csr merge --dtype $dt --reps 200
  echo "== lap $dt group"; SPMV_CSR_FLAT=0 python tools/exp.py lap4096 csr --dtype $dt --reps 200
done
echo "== rmat pipe"; python tools/exp.py rmat24 merge --reps 50
echo "== rmat persist"; SPMV_MERGE_VARIANT=1 python tools/exp.py rmat24 merge --reps 50
ncu --set full --clock-control none --import-source on -k regex:'k_(csr_flat|merge_pipe)' -c 2 -o gpurun_out/ncu_flat_pipe python tools/exp.py lap4096 csr merge --reps 1 > /dev/null 2>&1
