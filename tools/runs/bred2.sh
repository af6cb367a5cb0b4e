mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "inplace or direct_transport" > gpurun_out/bred2_parity.log 2>&1; tail -2 gpurun_out/bred2_parity.log
O=gpurun_out/bred2.jsonl
: > $O
SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 >> $O 2>&1
SMB_OPTS="bulkred=0" SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 >> $O 2>&1
SMB_INPLACE=1 SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 >> $O 2>&1
cat $O
