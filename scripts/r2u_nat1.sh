j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["roofline"]["kernel_norm_ms"], d["clocks"]["sm_mhz"])'
for r in 1 2 3; do
echo "base $(UC_LIB_PATH=build/ab/lib_base.so timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c "$j")"
echo "nat1 $(UC_LIB_PATH=build/ab/lib_nat1.so timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c "$j")"
done
