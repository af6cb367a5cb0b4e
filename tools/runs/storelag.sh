mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/storelag.jsonl
: > $O
for c in allgather reducescatter allreduce; do
for sl in 1 2; do
SMB_COLL=$c SMB_OPTS="storelag=$sl" SMB_INST=1,4 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w8s2t24576 >> $O 2>&1
done
SMB_COLL=$c SMB_OPTS="ring=1" SMB_INST=1,4 timeout 300 python tools/sm_budget.py 256 w16s2t24576 >> $O 2>&1
done
cat $O
