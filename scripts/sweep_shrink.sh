#!/bin/bash
# chunk-shrink sweep (rows off the first/last row chunk) at the bench workload: GLUPS + halo hidden fraction
OUT=gpurun_out/shrink; mkdir -p $OUT
for spec in "$@"; do
  sh=${spec%%|*}; a=${spec#*|}
  if [ "$sh" = "-" ]; then unset UC_CHUNK_SHRINK; else export UC_CHUNK_SHRINK=$sh; fi
  r=$(timeout 300 python bench.py --steps 5 --warmup 3 --halo-only $a 2>>$OUT/err.txt | tail -1)
  python - "$spec" "$r" <<'PY' | tee -a $OUT/sweep.txt
import json, sys
a, r = sys.argv[1], sys.argv[2]
try:
    d = json.loads(r); rf = d["roofline"]; h = d["halo"]
    print(f"shrink {a:30s} GLUPS={d['value']:8.1f} kernel_ms={rf['kernel_ms']:.4f} hidden={h['hidden_fraction']} full={h['t_full_ms']} comp={h['t_compute_ms']} xchg={h['t_xchg_ms']}")
except Exception as e:
    print(f"shrink {a:30s} FAILED {r[:300]}")
PY
done
