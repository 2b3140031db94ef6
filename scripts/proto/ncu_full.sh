mkdir -p gpurun_out/proto
ncu --set full --clock-control none --import-source on -k regex:"proto_kernel|jacobi_t_kernel" -s 2 -c 1 -o gpurun_out/proto/ta9 scripts/proto/bin/bm_T6_G2_M256_B2_ta9 16384 16384 7 9 0 ta9 > gpurun_out/proto/ncu_ta9.log 2>&1
PROTO_SHRINK=0 ncu --set full --clock-control none --import-source on -k regex:"proto_kernel|jacobi_t_kernel" -s 2 -c 1 -o gpurun_out/proto/full scripts/proto/bin/bm_T6_G2_M256_B2_full 16384 16384 7 9 0 full > gpurun_out/proto/ncu_full.log 2>&1
tail -1 gpurun_out/proto/ncu_full.log
