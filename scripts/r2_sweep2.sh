# sweeps at the current product kernel (bench --no-extras; 16384^2 per GPU unless stated)
T=${1:-sw2}
mkdir -p gpurun_out/$T
o=gpurun_out/$T/sweep.txt
j='import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"], d.get("halo") and d["halo"]["hidden_fraction"])'
for sh in 80 120 160 200 240; do echo "T=6 shrink=$sh $(UC_CHUNK_SHRINK=$sh timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
for t in 4 5 7 8; do echo "T=$t $(timeout 300 python bench.py --no-extras --steps 10 --tile-rows $t 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
for ny in 2048 4096 8192; do echo "ny=$ny $(timeout 300 python bench.py --ny-per-gpu $ny --halo-only --steps 20 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
for hp in 0,0 1,0 0,1 1,1; do echo "host $hp $(timeout 300 python bench.py --mode host --host-path $hp --no-extras --steps 5 2>&1 | tail -1 | python -c "$j" 2>&1)" >> $o; done
timeout 600 python benchmarks/p2p_sweep.py --vr 2 --scale 0.02 --max-bytes 4194304 > gpurun_out/$T/p2p_vr2.jsonl 2>&1; echo "p2p rc=$?" >> $o
cat $o
