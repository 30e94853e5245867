set -x
python -m pytest tests -m gpu -x -q -k "csr" 2>&1 | tail -3
python tools/exp.py lap4096 csr csr:vector_width=4 --reps 100
SPMV_CSR_FLAT=0 python tools/exp.py lap4096 csr --reps 100
python tools/exp.py lap4096 csr --dtype f32 --reps 100
SPMV_CSR_FLAT=0 python tools/exp.py lap4096 csr --dtype f32 --reps 100
