mkdir -p gpurun_out/trace5
o=gpurun_out/trace5/trace.txt
for sh in 160 240 320; do echo "== ring 16384 T=8 shrink $sh" >> $o; UC_CHUNK_SHRINK=$sh UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py >> $o 2>&1; done
j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"], d.get("halo") and d["halo"]["hidden_fraction"])'
for sh in 120 160 200 240 320; do echo "bench T=8 shrink=$sh $(UC_CHUNK_SHRINK=$sh timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
for ny in 2048 4096; do for d in 0 3 10; do echo "ny=$ny inject ${d}us $(timeout 300 python bench.py --ny-per-gpu $ny --halo-only --steps 20 --inject-delay-us $d 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done; done
cat $o
