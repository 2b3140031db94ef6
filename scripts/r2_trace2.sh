mkdir -p gpurun_out/trace2
o=gpurun_out/trace2/trace.txt
for sh in 320 160 0; do echo "== ring 16384 shrink $sh (gpu-scope flags)" >> $o; UC_CHUNK_SHRINK=$sh UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py >> $o 2>&1; done
echo "== ring 2048 default" >> $o; UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py --ny 2048 >> $o 2>&1
for sh in 320 160 80 0; do echo "bench shrink $sh: $(UC_CHUNK_SHRINK=$sh timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])' 2>&1)" >> $o; done
for ny in 2048 4096; do for sh in 0 80 160; do echo "ny $ny shrink $sh: $(UC_CHUNK_SHRINK=$sh timeout 300 python bench.py --ny-per-gpu $ny --halo-only --steps 20 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["halo"]["hidden_fraction"])' 2>&1)" >> $o; done; done
cat $o
