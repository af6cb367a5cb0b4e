mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/l2hint.jsonl
: > $O
for h in 1 0; do
for c in allgather allreduce; do
SMB_COLL=$c SMB_OPTS="l2hint=$h" SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 >> $O 2>&1
done
done
cat $O
