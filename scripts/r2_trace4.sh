mkdir -p gpurun_out/trace4
o=gpurun_out/trace4/trace.txt
echo "== ring 16384 default, per-warp DIRI" >> $o; UC_LIB_PATH=build/ab/lib_trace.so timeout 120 python scripts/trace_rounds.py >> $o 2>&1
for i in 1 2; do echo "bench default: $(timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])' 2>&1)" >> $o; done
cat $o
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "multi_step or jacobi or fullsize" > gpurun_out/trace4/pytest.log 2>&1; echo pytest_rc=$?; tail -3 gpurun_out/trace4/pytest.log
