#!/bin/bash
# Full GPU session: tests, smoke, ncu launch list + full capture of the dominant kernel, bench.
TAG=${1:-r1d}
OUT=gpurun_out/$TAG
mkdir -p $OUT
export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1; echo "build rc=$?" >> $OUT/build.txt
timeout 1800 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.txt
tail -5 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?" >> $OUT/smoke.txt
tail -2 $OUT/smoke.txt
timeout 600 python bench.py --steps 10 --warmup 3 > $OUT/bench.txt 2>&1; echo "bench rc=$?" >> $OUT/bench.txt
tail -3 $OUT/bench.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 --no-extras > $OUT/launches_bench.txt 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 80 -c 1 \
  -o $OUT/prof python bench.py --steps 1 --warmup 3 --no-extras > $OUT/prof_bench.txt 2>&1
echo "full rc=$?"
# the N > 1 launch path (torchrun, one process per rank, CUDA IPC peers) on the one GPU of the box
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --same-device --steps 3 --warmup 3 --ny-per-gpu 8192 > $OUT/bench_2proc.txt 2>&1; echo "2proc rc=$?" >> $OUT/bench_2proc.txt
tail -2 $OUT/bench_2proc.txt | cut -c1-600
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > $OUT/bench_ref.txt 2>&1; echo "ref rc=$?" >> $OUT/bench_ref.txt
tail -2 $OUT/bench_ref.txt | cut -c1-600
# configs[2]'s per-GPU share at P = 8 (16384 x 2048 slab) on one GPU, with the halo leg
timeout 300 python bench.py --steps 10 --warmup 3 --ny-per-gpu 2048 --halo-only > $OUT/bench_slab2048.txt 2>&1; echo "slab rc=$?" >> $OUT/bench_slab2048.txt
tail -2 $OUT/bench_slab2048.txt | cut -c1-300
