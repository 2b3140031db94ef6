# run every prototype binary in scripts/proto/bin (16384^2, default chunking) and collect JSON lines
cd "$(dirname "$0")"
mkdir -p ../../gpurun_out/proto
for b in bin/*; do timeout 60 ./$b 16384 16384 >> ../../gpurun_out/proto/wide.jsonl 2>&1 || echo "{\"bin\": \"$b\", \"rc\": $?}" >> ../../gpurun_out/proto/wide.jsonl; done
cat ../../gpurun_out/proto/wide.jsonl
