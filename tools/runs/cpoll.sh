# combine warps: one polling warp + named barrier (cpoll=1) vs all warps polling
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/cpoll.jsonl
: > $O
SMB_INST=1,4,8,12,18 timeout 600 python tools/sm_budget.py 256 w16s2t24576 w8s2t24576 >> $O 2>&1
SMB_OPTS="cpoll=1" SMB_INST=1,4,8,12,18 timeout 600 python tools/sm_budget.py 256 w16s2t24576 w8s2t24576 w32s2t24576 >> $O 2>&1
SMB_COLL=reducescatter SMB_OPTS="cpoll=1" SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 >> $O 2>&1
RESCCL_CPOLL=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/cpoll_parity.log 2>&1; tail -2 gpurun_out/cpoll_parity.log >> $O
cat $O
