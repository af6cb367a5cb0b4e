mkdir -p gpurun_out
B=build/per_sm_bw
O=gpurun_out/per_sm.jsonl
: > $O
for nb in 8 32 148; do
  for m in 0 1; do for t in 256 512 1024; do for u in 4 8 16; do timeout 20 $B $m $nb $t $u 0 64 >> $O; done; done; done
  for m in 2 3; do for t in 256 512; do for s in 4 8 16; do for T in 8192 12288 16384 24576; do
    if [ $((s*2*T)) -le 200000 ]; then timeout 20 $B $m $nb $t $s $T 64 >> $O; fi; done; done; done; done
done
cat $O
