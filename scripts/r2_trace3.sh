mkdir -p gpurun_out/trace3
o=gpurun_out/trace3/trace.txt
echo "== ring 16384 default (160)" >> $o; UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py >> $o 2>&1
echo "== chain 16384 default" >> $o; UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py --topology dirichlet >> $o 2>&1
for i in 1 2; do echo "bench default: $(timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])' 2>&1)" >> $o; done
cat $o
