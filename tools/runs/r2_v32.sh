# r02: the 96-CTA bench default: element-wise full-size parity, bench line, ncu launch list + full capture
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -q -m gpu > gpurun_out/r2v32_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v32_pytest.log
tail -2 gpurun_out/r2v32_pytest.log
timeout 900 python bench.py > gpurun_out/r2v32_bench.json 2> gpurun_out/r2v32_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2v32_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --inplace-steps 0 --sweep "" --tuned-sweep "" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/r2v32_prof python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --inplace-steps 0 --sweep "" --tuned-sweep "" > gpurun_out/r2v32_ncu.log 2>&1
ncu -i gpurun_out/r2v32_prof.ncu-rep --page raw --csv > gpurun_out/r2v32_prof_raw.csv 2>/dev/null
ncu -i gpurun_out/r2v32_prof.ncu-rep --page details --csv > gpurun_out/r2v32_prof_details.csv 2>/dev/null
rm -f gpurun_out/r2v32_prof.ncu-rep
cat gpurun_out/r2v32_bench.json | cut -c1-1500
