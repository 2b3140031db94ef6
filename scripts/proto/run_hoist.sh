cd "$(dirname "$0")"; mkdir -p ../../gpurun_out/proto; out=../../gpurun_out/proto/hoist.jsonl
for r in 1 2; do
for h in 0 2 3 4 8; do timeout 60 ./bin/bm_T8_h$h 16384 16384 7 9 0 T8h$h >> $out 2>&1; done
for h in 0 2 3 6; do timeout 60 ./bin/bm_T6_h$h 16384 16384 7 9 0 T6h$h >> $out 2>&1; done
done
cat $out
