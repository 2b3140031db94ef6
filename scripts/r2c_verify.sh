# round-2 re-entry verification of HEAD: smoke, GPU tests, bench line
set -x
T=${1:-r2c}
mkdir -p gpurun_out/$T
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/$T/smi.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/$T/pytest.log 2>&1; echo pytest_rc=$?
tail -5 gpurun_out/$T/pytest.log
timeout 900 python bench.py > gpurun_out/$T/bench.log 2>&1; echo bench_rc=$?
tail -c 3000 gpurun_out/$T/bench.log
