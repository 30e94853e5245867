# round-end evidence (one call): parity suite, bench lines, ncu captures + summaries, sanitizers,
# then the regenerated sweep (configs[3]) and R-MAT27 check with the final kernels
bash tools/gpu/round_end.sh
bash tools/gpu/sanitize.sh > gpurun_out/sanitize.txt 2>&1
bash tools/gpu/regen_results.sh
