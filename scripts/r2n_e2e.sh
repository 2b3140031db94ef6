# e2e leg with 2/3/4 solvers in flight (bench default carries 3)
set -x
O=gpurun_out/e2e; mkdir -p $O
for S in 2 3 4; do timeout 600 python bench.py --steps 10 --e2e-streams $S > $O/bench_s$S.log 2>&1; tail -1 $O/bench_s$S.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["e2e"])'; done
