python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "coo or hyb" 2>&1 | tail -3
for d in f64 f32; do for p in 0 1; do SPMV_COO_PIPE=$p timeout 300 python tools/fmt_time.py lap4096 $d coo,csr5 --tag pipe$p; done; done
for p in 0 1; do SPMV_COO_PIPE=$p timeout 300 python tools/fmt_time.py rmat24 f64 coo,csr5 --tag pipe$p; done
