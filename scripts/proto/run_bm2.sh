# block-ring march prototypes, explicit (binary, consumer warps, stages) list
cd "$(dirname "$0")"
mkdir -p ../../gpurun_out/proto
out=../../gpurun_out/proto/bm_${1:-run}.jsonl
while read b w ns; do
  [ -z "$b" ] && continue
  timeout 60 ./bin/$b 16384 16384 $w $ns 0 $b >> $out 2>&1 || echo "{\"bin\": \"$b\", \"ns\": $ns, \"rc\": $?}" >> $out
done < ${LIST:-list.txt}
cat $out
