cd "$(dirname "$0")"
mkdir -p ../../gpurun_out/proto; out=../../gpurun_out/proto/bm_full2.jsonl
for b in bm_T6_G2_M256_B2_full bm_T6_G2_M256_B2_fullni; do
  for sh in 0 160 320; do PROTO_SHRINK=$sh timeout 60 ./bin/$b 16384 16384 7 9 0 $b >> $out 2>&1; done
done
timeout 60 ./bin/bm_T6_G2_M256_B2_ta9 16384 16384 7 9 0 ta9 >> $out 2>&1
cat $out
