# pairwise acc_sq: bench x2 (kernel_norm_ms), full GPU suite
set -x
O=gpurun_out/norm; mkdir -p $O
j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["roofline"]["kernel_norm_ms"], d["clocks"]["sm_mhz"])'
for i in 1 2; do echo "bench $(timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c "$j")"; done
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest_rc=$?
tail -3 $O/pytest.log
