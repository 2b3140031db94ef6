# depth sweep of the final build (pair frame + scaled march) and an ncu capture of the norm launch
set -x
O=gpurun_out/tsweep; mkdir -p $O
j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["roofline"]["kernel_norm_ms"], d["config"]["launch"]["grid"], d["clocks"]["sm_mhz"])'
for t in 5 6 7 8; do echo "T=$t $(timeout 300 python bench.py --no-extras --steps 10 --tile-rows $t 2>&1 | tail -1 | python -c "$j")"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 0 -c 1 -o $O/norm python bench.py --steps 1 --warmup 3 --no-extras > $O/ncu_norm.log 2>&1; echo ncu_rc=$?
