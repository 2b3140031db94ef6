mkdir -p gpurun_out/proto
ncu --set full --import-source on -k regex:proto_kernel -s 2 -c 1 -o gpurun_out/proto/grp9 scripts/proto/bin/bm_T6_G2_M256_B2_grp9 16384 16384 7 9 0 grp9 > gpurun_out/proto/ncu_grp9.log 2>&1
ncu --set full --import-source on -k regex:proto_kernel -s 2 -c 1 -o gpurun_out/proto/old scripts/proto/bin/bm_T6_G2_M256_B2_old 16384 16384 7 8 0 old > gpurun_out/proto/ncu_old.log 2>&1
tail -2 gpurun_out/proto/ncu_grp9.log
