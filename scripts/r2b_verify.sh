# round-2 verification pass: GPU tests, smoke (P = 1), bench (default + spawned 2 ranks on one GPU),
# reference arm, ncu launch list of the smoke run
set -x
mkdir -p gpurun_out/r2b
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2b/smoke.log 2>&1; echo smoke_rc=$?
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2b/launches_smoke.csv python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2b/ncu_smoke.log 2>&1; echo ncu_smoke_rc=$?
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/r2b/pytest.log 2>&1; echo pytest_rc=$?
tail -5 gpurun_out/r2b/pytest.log
timeout 600 python bench.py > gpurun_out/r2b/bench.log 2>&1; echo bench_rc=$?
timeout 300 python bench.py --gpus 2 --same-device --no-extras --steps 3 --warmup 3 > gpurun_out/r2b/bench_spawn2.log 2>&1; echo spawn_rc=$?
timeout 300 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r2b/bench_ref.log 2>&1; echo ref_rc=$?
tail -c 1500 gpurun_out/r2b/bench.log
