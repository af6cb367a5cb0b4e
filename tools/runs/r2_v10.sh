mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2v10_smoke.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r2v10_pytest_all.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v10_pytest_all.log
timeout 900 python bench.py > gpurun_out/r2v10_bench.json 2> gpurun_out/r2v10_bench.err
tail -5 gpurun_out/r2v10_pytest_all.log; cat gpurun_out/r2v10_bench.json; tail -3 gpurun_out/r2v10_bench.err
