# round-2 final verification of the product: smoke, full GPU suite, bench line, host comparator,
# thin slab + injected flag latency, spawned ranks, reference arm, P2P sweep machinery, ncu, sanitizers
set -x
T=${1:-r2final}
O=gpurun_out/$T
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke_rc=$?
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest_rc=$?
tail -3 $O/pytest.log
timeout 900 python bench.py > $O/bench.log 2>&1; echo bench_rc=$?
timeout 300 python bench.py --no-extras --steps 10 > $O/bench2.log 2>&1
timeout 300 python bench.py --mode host --host-path 1,1 --no-extras --steps 10 > $O/bench_host11.log 2>&1
timeout 300 python bench.py --mode host --host-path 0,0 --no-extras --steps 5 > $O/bench_host00.log 2>&1
for ny in 2048 16384; do for d in 0 3 10; do timeout 300 python bench.py --ny-per-gpu $ny --halo-only --steps 10 --inject-delay-us $d > $O/halo_${ny}_d$d.log 2>&1; done; done
timeout 300 python bench.py --ny-per-gpu 2048 --no-extras --steps 20 > $O/bench_slab2048.log 2>&1
timeout 300 python bench.py --gpus 2 --same-device --no-extras --steps 3 --warmup 3 > $O/bench_spawn2.log 2>&1; echo spawn_rc=$?
timeout 300 python bench.py --impl reference --steps 10 --warmup 3 > $O/bench_ref.log 2>&1; echo ref_rc=$?
timeout 600 python benchmarks/p2p_sweep.py --vr 2 --scale 0.1 --max-bytes 16777216 --no-nccl > $O/p2p_sweep.jsonl 2>$O/p2p_sweep.err; echo p2p_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 3 --no-extras > $O/ncu_launch.log 2>&1; echo ncu_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 4 -c 1 -o $O/prof python bench.py --steps 1 --warmup 3 --no-extras > $O/ncu_full.log 2>&1; echo ncu_full_rc=$?
for t in memcheck synccheck racecheck; do UC_SANITIZE_T6_ONLY=1 timeout 1200 compute-sanitizer --tool $t --error-exitcode 9 python scripts/sanitize_run.py > $O/san_$t.log 2>&1; echo "$t rc=$?" >> $O/san_rc.txt; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|SANITIZE_RUN_DONE" $O/san_$t.log >> $O/san_rc.txt; done
cat $O/san_rc.txt
for f in $O/bench*.log $O/halo_*.log; do echo "$f $(tail -1 $f | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d.get("value"), d.get("roofline",{}).get("kernel_ms"), (d.get("halo") or {}).get("hidden_fraction"), d.get("clocks",{}).get("sm_mhz"))' 2>&1)"; done
