# scaled march: new parity tests first, A/B bench (scaled product vs unscaled PQ vs round-2 natural), full GPU suite
set -x
T=${1:-sc}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
timeout 600 python -m pytest tests/test_gpu_multi_step.py -q -p no:cacheprovider -k scaled > gpurun_out/$T/pytest_scaled.log 2>&1; echo pytest_scaled_rc=$?
tail -15 gpurun_out/$T/pytest_scaled.log
for i in 1 2; do
  timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_sc_$i.log 2>&1
  UC_LIB_PATH=build/ab/lib_unscaled.so timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_pq_$i.log 2>&1
  UC_LIB_PATH=build/ab/lib_pq0.so timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_nat_$i.log 2>&1
done
for f in gpurun_out/$T/bench_*.log; do echo "$f $(tail -1 $f | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"], d.get("scaled_march_reruns"))' 2>&1)"; done
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; echo pytest_rc=$?
tail -15 gpurun_out/$T/pytest.log
