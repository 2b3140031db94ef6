mkdir -p gpurun_out/trace
o=gpurun_out/trace/trace.txt
for sh in 320 0; do echo "== ring 16384 shrink $sh" >> $o; UC_CHUNK_SHRINK=$sh UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py >> $o 2>&1; done
echo "== chain 16384 default" >> $o; UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py --topology dirichlet >> $o 2>&1
echo "== ring 2048 default" >> $o; UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py --ny 2048 >> $o 2>&1
cat $o
cd scripts/proto; for h in 2000 20000 1000000; do timeout 60 ./bin/bm_T6_G2_M256_B2_h$h 16384 16384 7 9 0 hint$h >> ../../gpurun_out/trace/hint.jsonl 2>&1; done; timeout 60 ./bin/bm_T6_G2_M256_B2_ta9 16384 16384 7 9 0 ta9 >> ../../gpurun_out/trace/hint.jsonl 2>&1; cat ../../gpurun_out/trace/hint.jsonl
