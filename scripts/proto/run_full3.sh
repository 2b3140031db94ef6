cd "$(dirname "$0")"
mkdir -p ../../gpurun_out/proto; out=../../gpurun_out/proto/bm_full3.jsonl
for b in bm_T6_G2_M256_B2_full bm_T6_G2_M256_B2_fullw bm_T6_G2_M256_B2_fullwni bm_T6_G2_M256_B2_ta9; do
  for sh in 0 320; do PROTO_SHRINK=$sh timeout 60 ./bin/$b 16384 16384 7 9 0 $b >> $out 2>&1; done
done
cat $out
