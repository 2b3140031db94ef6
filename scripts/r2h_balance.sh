# balanced chunks: new parity tests, A/B bench (balanced vs static chunks), full GPU suite
set -x
T=${1:-bal}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
timeout 900 python -m pytest tests/test_gpu_multi_step.py -q -p no:cacheprovider -k "balance or scaled" > gpurun_out/$T/pytest_bal.log 2>&1; echo pytest_bal_rc=$?
tail -25 gpurun_out/$T/pytest_bal.log
for i in 1 2; do
  timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_bal_$i.log 2>&1
  timeout 300 python bench.py --no-extras --steps 10 --no-balance > gpurun_out/$T/bench_static_$i.log 2>&1
done
timeout 300 python bench.py --no-extras --steps 30 > gpurun_out/$T/bench_bal_30.log 2>&1
for f in gpurun_out/$T/bench_*.log; do echo "$f $(tail -1 $f | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["roofline"]["kernel_share_of_step"], d["clocks"]["sm_mhz"], d.get("scaled_march_reruns"))' 2>&1)"; done
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; echo pytest_rc=$?
tail -15 gpurun_out/$T/pytest.log
