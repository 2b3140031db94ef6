# in-warp ring feed (8 consumer warps, no producer warp) vs the producer-warp build: smoke, parity subset, bench A/B
set -x
T=${1:-iw}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
tail -2 gpurun_out/$T/smoke.log
for i in 1 2; do
  timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_iw_$i.log 2>&1
  UC_LIB_PATH=build/ab/lib_prodwarp.so timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_pw_$i.log 2>&1
done
for f in gpurun_out/$T/bench_*.log; do echo "$f $(tail -1 $f | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["config"]["launch"], d["clocks"]["sm_mhz"])' 2>&1)"; done
timeout 1500 python -m pytest tests/test_gpu_multi_step.py -x -q -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; echo pytest_rc=$?
tail -5 gpurun_out/$T/pytest.log
