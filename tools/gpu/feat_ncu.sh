python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:^k_features -s 3 -c 1 -o gpurun_out/feat_lap python tools/feat_time.py lap4096 > gpurun_out/ncu1.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:^k_features -s 3 -c 1 -o gpurun_out/feat_rmat python tools/feat_time.py rmat24 > gpurun_out/ncu2.log 2>&1
ls -la gpurun_out
