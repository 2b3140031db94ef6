# after the balance default flip: balance/scaled parity tests, smoke, default bench x2
set -x
T=${1:-chk}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
timeout 900 python -m pytest tests/test_gpu_multi_step.py -q -p no:cacheprovider -k "balance or scaled" > gpurun_out/$T/pytest_bal.log 2>&1; echo pytest_bal_rc=$?
tail -5 gpurun_out/$T/pytest_bal.log
for i in 1 2; do timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_$i.log 2>&1; tail -1 gpurun_out/$T/bench_$i.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])'; done
