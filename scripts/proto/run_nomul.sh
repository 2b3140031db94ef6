cd "$(dirname "$0")"; mkdir -p ../../gpurun_out/proto; out=../../gpurun_out/proto/nomul.jsonl
for b in cur nomul cur nomul; do timeout 60 ./bin/bm_T6_G2_M256_B2_$b 16384 16384 7 9 0 $b >> $out 2>&1; done; cat $out
