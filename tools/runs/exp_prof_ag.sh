mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/smb4.jsonl
: > $O
for o in "" "l2hint=0"; do
  SMB_COLL=allgather SMB_INST=4 SMB_OPTS="$o" timeout 120 python tools/sm_budget.py 256 one >> $O 2>> gpurun_out/smb4.err
  SMB_COLL=reducescatter SMB_INST=4 SMB_OPTS="$o" timeout 120 python tools/sm_budget.py 256 one >> $O 2>> gpurun_out/smb4.err
done
OPTS="instances=4 nwarps=16 tmastages=4 tmatile=12288 chunkbytes=33554432 fifodepth=2 direct=1"
timeout 300 ncu --set full --clock-control none --import-source on -k regex:resccl -s 1 -c 1 -o gpurun_out/prof_ag4 python tools/one_coll.py allgather 256 "$OPTS" 2 > gpurun_out/prof_ag4.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:resccl -s 1 -c 1 -o gpurun_out/prof_rs4 python tools/one_coll.py reducescatter 256 "$OPTS" 2 > gpurun_out/prof_rs4.log 2>&1
timeout 300 ncu --set full --clock-control none -k regex:k_tma -s 1 -c 1 -o gpurun_out/prof_mb2 build/per_sm_bw 2 32 256 4 24576 64 > gpurun_out/prof_mb2.log 2>&1
for f in prof_ag4 prof_rs4 prof_mb2; do
  ncu -i gpurun_out/$f.ncu-rep --page details --csv > gpurun_out/${f}_details.csv 2>/dev/null
  ncu -i gpurun_out/$f.ncu-rep --page raw --csv > gpurun_out/${f}_raw.csv 2>/dev/null
  ncu -i gpurun_out/$f.ncu-rep --page source --csv > gpurun_out/${f}_source.csv 2>/dev/null
done
cat $O
