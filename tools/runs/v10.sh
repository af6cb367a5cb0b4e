mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_v10.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v10.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_v10.log
python bench.py > gpurun_out/bench_v10.json 2> gpurun_out/bench_v10.err
SMB_INPLACE=1 SMB_INST=1,4,8,12,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 > gpurun_out/sm_budget_inplace_v10.jsonl 2>&1
tail -3 gpurun_out/pytest_gpu_v10.log; cat gpurun_out/bench_v10.json; cat gpurun_out/sm_budget_inplace_v10.jsonl
