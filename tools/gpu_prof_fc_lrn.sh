# ncu --set full of the FC and LRN+pool kernels (B=256 and B=1), source-level
cd $GRAFT_REPO_ROOT
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:"fc_tc|lrn_reg" -s 10 -c 5 -o gpurun_out/full_fclrn_b256 python bench.py --minimal --steps 1 --warmup 3 > gpurun_out/ncu_b256.log 2>&1
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:"fc_tc|conv_tc|stage|lrn" -s 26 -c 13 -o gpurun_out/full_b1 python bench.py --minimal --steps 1 --warmup 3 --batch 1 > gpurun_out/ncu_b1.log 2>&1
ls -la gpurun_out
