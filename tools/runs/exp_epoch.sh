mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/exp_epoch.jsonl
: > $O
for c in reducescatter allgather allreduce; do
  SMB_COLL=$c SMB_INST=4 timeout 120 python tools/sm_budget.py 256 one >> $O 2>&1
done
SMB_INST=1,4,8,12,18 timeout 300 python tools/sm_budget.py 256 one two >> $O 2>&1
SMB_INST=24,30,37 timeout 300 python tools/sm_budget.py 256 two >> $O 2>&1
cat $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/parity_epoch.log 2>&1; tail -2 gpurun_out/parity_epoch.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_epoch.log 2>&1; tail -3 gpurun_out/pytest_gpu_epoch.log
