O=gpurun_out/stages; mkdir -p $O
j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])'
for r in 1 2; do for st in 9 18 27; do echo "stages=$st $(timeout 300 python bench.py --no-extras --steps 10 --stages $st 2>&1 | tail -1 | python -c "$j")"; done; done
