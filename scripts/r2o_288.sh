# 8 consumer warps + producer per block (288 threads, 112 registers) at T = 6/7/8 vs the product (256 threads, T = 8)
set -x
O=gpurun_out/b288; mkdir -p $O
j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["config"]["launch"], d["clocks"]["sm_mhz"])'
for i in 1 2; do
  echo "prod T8 $(timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c "$j")"
  for t in 7 6; do echo "288 T$t $(UC_LIB_PATH=build/ab/lib_288.so timeout 300 python bench.py --no-extras --steps 10 --tile-rows $t 2>&1 | tail -1 | python -c "$j")"; done
done
echo "288 T8 $(UC_LIB_PATH=build/ab/lib_288.so timeout 300 python bench.py --no-extras --steps 10 --tile-rows 8 2>&1 | tail -1 | python -c "$j")"
echo "prod T7 $(timeout 300 python bench.py --no-extras --steps 10 --tile-rows 7 2>&1 | tail -1 | python -c "$j")"
