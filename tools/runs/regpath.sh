# register (LD/ST) path vs TMA engine per SM
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/regpath.jsonl
: > $O
SMB_OPTS="tma=0" SMB_INST=1,4,8,18 timeout 600 python tools/sm_budget.py 256 w16s2t24576 w32s2t24576 >> $O 2>&1
SMB_COLL=reducescatter SMB_OPTS="tma=0" SMB_INST=1,4 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w32s2t24576 >> $O 2>&1
SMB_COLL=allgather SMB_OPTS="tma=0" SMB_INST=1,4 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w32s2t24576 >> $O 2>&1
cat $O
