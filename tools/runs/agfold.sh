mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v11.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_v11.log
SMB_COLL=allgather SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w8s2t24576 > gpurun_out/agfold_smb.jsonl 2>&1
timeout 1200 python tools/sweep.py c2 > gpurun_out/sweep_c2_v11.jsonl 2>&1
tail -3 gpurun_out/pytest_gpu_v11.log; cat gpurun_out/agfold_smb.jsonl
