T=${1:-ab2}; mkdir -p gpurun_out/$T; o=gpurun_out/$T/ab.txt
j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["roofline"]["kernel_norm_ms"], d["clocks"]["sm_mhz"], d["roofline"]["launch_plan_per_step"][-3:])'
for r in 1 2; do
for t in 6 8; do echo "product T=$t $(timeout 300 python bench.py --no-extras --steps 10 --tile-rows $t 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
for t in 6; do echo "hoist62=6 T=$t $(UC_LIB_PATH=build/ab/lib_h66.so timeout 300 python bench.py --no-extras --steps 10 --tile-rows $t 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
done
for t in 7; do echo "product T=$t $(timeout 300 python bench.py --no-extras --steps 10 --tile-rows $t 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
cat $o
