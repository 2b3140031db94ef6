#!/bin/bash
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
for a in "$@"; do
  r=$(timeout 300 python benchmarks/cg_bench.py --cpu-iters 0 --steps 3 $a 2>>$OUT/err.txt | tail -1)
  python -c "
import json,sys
try:
  d=json.loads(sys.argv[2]); print(f'{sys.argv[1]:40s} it/s={d[\"value\"]:8.1f} ms/it={d[\"ms_per_iteration\"]:.4f} GB/s={d[\"roofline\"][\"achieved\"]:7.1f} frac={d[\"roofline\"][\"frac\"]:.3f}')
except Exception as e: print(sys.argv[1], 'FAILED', sys.argv[2][:200])
" "$a" "$r" | tee -a $OUT/sweep.txt
done
