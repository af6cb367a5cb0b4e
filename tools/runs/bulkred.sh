mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "inplace_tma" > gpurun_out/bulkred_parity.log 2>&1; tail -3 gpurun_out/bulkred_parity.log
O=gpurun_out/bulkred.jsonl
: > $O
for br in 0 1; do
SMB_INPLACE=1 SMB_OPTS="bulkred=$br" SMB_INST=1,4,8,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w8s2t24576 >> $O 2>&1
SMB_COLL=reducescatter SMB_INPLACE=1 SMB_OPTS="bulkred=$br" SMB_INST=1,4 timeout 300 python tools/sm_budget.py 256 w16s2t24576 >> $O 2>&1
done
cat $O
