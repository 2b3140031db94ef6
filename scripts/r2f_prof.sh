# profile the scaled march (launch list + ncu --set full of one <8,2> launch) and A/B: hoisted
# neighbour levels 0/4/8, ring stages 18
set -x
T=${1:-r2s}
mkdir -p gpurun_out/$T
timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench.log 2>&1; echo bench_rc=$?
for lib in h0 h4 h8; do UC_LIB_PATH=build/ab/lib_$lib.so timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_$lib.log 2>&1; done
timeout 300 python bench.py --no-extras --steps 10 --stages 18 > gpurun_out/$T/bench_st18.log 2>&1
timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_2.log 2>&1
for f in gpurun_out/$T/bench*.log; do echo "$f $(tail -1 $f | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"], d.get("scaled_march_reruns"))' 2>&1)"; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$T/launches.csv python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/$T/ncu_launch.log 2>&1; echo ncu_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 4 -c 1 -o gpurun_out/$T/prof python bench.py --steps 1 --warmup 3 --no-extras > gpurun_out/$T/ncu_full.log 2>&1; echo ncu_full_rc=$?
ls -la gpurun_out/$T
