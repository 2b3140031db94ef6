# per-block / per-SM timing of the T = 8 product launch (UC_TRACE build), then bench of the new default (hoist 8)
set -x
mkdir -p gpurun_out/trace6
UC_LIB_PATH=build/ab/lib_trace.so timeout 300 python scripts/trace_rounds.py > gpurun_out/trace6/trace.txt 2>&1; echo trace_rc=$?
cat gpurun_out/trace6/trace.txt
for i in 1; do timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/trace6/bench_$i.log 2>&1; tail -1 gpurun_out/trace6/bench_$i.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"], d.get("scaled_march_reruns"))'; done
