mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/smb3.jsonl
: > $O
for coll in allreduce reducescatter allgather; do
  SMB_COLL=$coll SMB_INST=1,4,8,18 timeout 300 python tools/sm_budget.py 256 one two >> $O 2>> gpurun_out/smb3.err
done
SMB_INST=24,30,37 timeout 300 python tools/sm_budget.py 256 two >> $O 2>> gpurun_out/smb3.err
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/parity3.log 2>&1; tail -2 gpurun_out/parity3.log
cat $O
