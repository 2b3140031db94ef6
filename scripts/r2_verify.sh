# round-2 verification pass (usage: bash scripts/r2_verify.sh <tag> [pytest -k expr]):
# GPU tests, smoke, bench line, ncu launch list of a short bench
set -x
T=${1:-r2}; K=${2:-}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
if [ -n "$K" ]; then timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "$K" > gpurun_out/$T/pytest.log 2>&1; else timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; fi; echo pytest_rc=$?
tail -3 gpurun_out/$T/pytest.log
timeout 600 python bench.py > gpurun_out/$T/bench.log 2>&1; echo bench_rc=$?
timeout 300 python bench.py --mode host --no-extras --steps 5 > gpurun_out/$T/bench_host.log 2>&1; echo bench_host_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$T/launches.csv python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/$T/ncu_launch.log 2>&1; echo ncu_rc=$?
tail -c 600 gpurun_out/$T/bench.log
