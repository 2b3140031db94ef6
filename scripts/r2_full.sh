# full round-2 verification: smoke, GPU tests, bench line, sanitizer on the deep kernels, ncu
set -x
T=${1:-r2full}
mkdir -p gpurun_out/$T
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; echo pytest_rc=$?
tail -5 gpurun_out/$T/pytest.log
timeout 900 python bench.py > gpurun_out/$T/bench.log 2>&1; echo bench_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$T/launches.csv python bench.py --steps 2 --warmup 3 --no-extras > gpurun_out/$T/ncu_launch.log 2>&1; echo ncu_rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 4 -c 1 -o gpurun_out/$T/t8 python bench.py --steps 1 --warmup 3 --no-extras > gpurun_out/$T/ncu_full.log 2>&1; echo ncu_full_rc=$?
for t in memcheck synccheck racecheck; do UC_SANITIZE_T6_ONLY=1 timeout 900 compute-sanitizer --tool $t python scripts/sanitize_run.py > gpurun_out/$T/san_$t.log 2>&1; echo "$t rc=$?" >> gpurun_out/$T/san_rc.txt; done
cat gpurun_out/$T/san_rc.txt
tail -c 800 gpurun_out/$T/bench.log
