mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 900 python -m pytest tests/test_gpu_parity_r2.py tests/test_gpu_parity.py -q -x -m gpu -k "tb_util or direct or graph" > gpurun_out/r2v9_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v9_pytest.log
timeout 600 python tools/tb_util.py 256 best > gpurun_out/r2v9_tbutil_best.jsonl 2> gpurun_out/r2v9_tbutil.err
timeout 600 python tools/tb_util.py 64 r01 > gpurun_out/r2v9_tbutil_r01.jsonl 2>> gpurun_out/r2v9_tbutil.err
tail -2 gpurun_out/r2v9_pytest.log; cat gpurun_out/r2v9_tbutil_best.jsonl | cut -c1-80; tail -3 gpurun_out/r2v9_tbutil.err
