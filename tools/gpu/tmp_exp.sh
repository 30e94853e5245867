for v in 1 2 3; do echo "PAIRS=$v"; SPMV_MERGE_PAIRS=$v timeout 60 python tools/exp.py lap4096 merge --reps 300 2>&1 | tail -1; SPMV_MERGE_PAIRS=$v timeout 60 python tools/exp.py lap4096 merge --dtype f32 --reps 300 2>&1 | tail -1; done
SPMV_MERGE_PAIRS=3 timeout 300 python -m pytest tests -m gpu -x -q -k "merge" -p no:cacheprovider 2>&1 | tail -1
