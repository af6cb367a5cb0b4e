mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/smb2.jsonl
: > $O
for coll in allreduce reducescatter allgather; do
  for bo in "" "backoff=0"; do
    SMB_COLL=$coll SMB_INST=1,4,8 SMB_OPTS="$bo" timeout 300 python tools/sm_budget.py 256 one two >> $O 2>> gpurun_out/smb2.err
  done
done
SMB_INST=1,4,8 SMB_OPTS="backoff=0 tmamin=1024" SMB_CB=4194304 timeout 300 python tools/sm_budget.py 256 one >> $O 2>> gpurun_out/smb2.err
cat $O
