#!/bin/bash
# Kernel A/B sweep at the bench workload.
# Usage: bash scripts/sweep.sh TAG "libname|bench args" ...   (libname "-" = product build)
TAG=$1; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
for spec in "$@"; do
  lib=${spec%%|*}; a=${spec#*|}
  if [ "$lib" = "-" ]; then unset UC_LIB_PATH; else export UC_LIB_PATH=build/ab/$lib.so; fi
  r=$(timeout 300 python bench.py --steps 5 --warmup 3 --no-extras $a 2>>$OUT/err.txt | tail -1)
  python - "$spec" "$r" <<'PY' | tee -a $OUT/sweep.txt
import json, sys
a, r = sys.argv[1], sys.argv[2]
try:
    d = json.loads(r)
    rf = d["roofline"]
    print(f"{a:45s} GLUPS={d['value']:8.1f} kernel_ms={rf['kernel_ms']:.4f} GB/s={rf['achieved']:7.1f} frac={rf['frac']:.4f} norm_ms={rf['kernel_norm_ms']:.4f} launch={d['config']['launch']}")
except Exception as e:
    print(f"{a:45s} FAILED {r[:200]}")
PY
done
unset UC_LIB_PATH
