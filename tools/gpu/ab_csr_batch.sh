python -c "import __graft_entry__ as g; g.build()" >/dev/null
for v in base vA vB vC vD; do
  L=paper_conf_ipps_nisassvs18_b200/libspmv.so; [ $v != base ] && L=build/variants/$v/libspmv.so
  for d in f64 f32; do SPMV_LIB_PATH=$L python tools/exp_csrw.py rmat24 $d 0 | sed "s/^/$v /" | cut -c1-110; done
  SPMV_LIB_PATH=$L python tools/exp_csrw.py u2048 f64 0 | sed "s/^/$v /" | cut -c1-110
done
