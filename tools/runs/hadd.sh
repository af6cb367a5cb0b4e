mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/hadd_parity.log 2>&1; tail -3 gpurun_out/hadd_parity.log
O=gpurun_out/hadd.jsonl
: > $O
SMB_INST=1,4,8,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w8s2t24576 >> $O 2>&1
SMB_COLL=reducescatter SMB_INST=1,4 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w8s2t24576 >> $O 2>&1
cat $O
