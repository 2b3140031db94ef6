cd "$(dirname "$0")"; mkdir -p ../../gpurun_out/proto; out=../../gpurun_out/proto/gb.jsonl
for r in 1 2; do
timeout 60 ./bin/bm_T8_gb0 16384 16384 7 9 0 gb0_w7 >> $out 2>&1
timeout 60 ./bin/bm_T8_gb1 16384 16384 7 9 0 gb1_w7 >> $out 2>&1
timeout 60 ./bin/bm_T8_gb0 16384 16384 6 9 0 gb0_w6 >> $out 2>&1
timeout 60 ./bin/bm_T8_gb0 16384 16384 5 9 0 gb0_w5 >> $out 2>&1
timeout 60 ./bin/bm_T8_gb0 16384 16384 7 18 0 gb0_w7_ns18 >> $out 2>&1
done
cat $out
