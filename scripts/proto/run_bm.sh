# block-ring march prototypes: bin/bm_T<T>_M<maxthreads>_B<minblocks>; consumer warps = maxthreads/32 - 1
cd "$(dirname "$0")"
mkdir -p ../../gpurun_out/proto
out=../../gpurun_out/proto/bm_${1:-run}.jsonl
for b in bin/bm_*; do
  m=$(echo $b | sed 's/.*_M\([0-9]*\)_.*/\1/'); w=$((m / 32 - 1))
  for ns in ${NSLIST:-8}; do timeout 60 ./$b 16384 16384 $w $ns 0 $(basename $b) >> $out 2>&1 || echo "{\"bin\": \"$b\", \"rc\": $?}" >> $out; done
done
cat $out
