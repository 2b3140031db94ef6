# shrink / depth sweep of the product kernel (bench --no-extras, 16384^2, P = 1 ring)
T=${1:-sweep}
mkdir -p gpurun_out/$T
out=gpurun_out/$T/sweep.txt
for sh in 0 80 160 240 320; do
  r=$(UC_CHUNK_SHRINK=$sh timeout 300 python bench.py --no-extras --steps 10 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])' 2>&1)
  echo "T=6 shrink=$sh $r" >> $out
done
for t in 5 7 8; do
  r=$(timeout 300 python bench.py --no-extras --steps 10 --tile-rows $t 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])' 2>&1)
  echo "T=$t default shrink $r" >> $out
done
for ny in 2048 4096; do
  for sh in 0 40 80 160; do
    r=$(UC_CHUNK_SHRINK=$sh timeout 300 python bench.py --ny-per-gpu $ny --halo-only --steps 20 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["halo"]["hidden_fraction"], d["config"]["launch"])' 2>&1)
    echo "ny=$ny T=6 shrink=$sh $r" >> $out
  done
done
cat $out
