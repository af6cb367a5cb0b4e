# r02 first pass: new GPU tests, whole GPU suite, bench at 112 CTAs, latency probe, ncu of the bench kernel
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2v1_smoke.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity_r2.py tests/test_gpu_fullsize.py tests/test_gpu_multidevice.py -m gpu -q > gpurun_out/r2v1_pytest_new.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v1_pytest_new.log
timeout 1500 python -m pytest tests -m gpu -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r2v1_pytest_all.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v1_pytest_all.log
python bench.py > gpurun_out/r2v1_bench.json 2> gpurun_out/r2v1_bench.err
LAT_SIZES="[1024, 1048576, 16777216]" timeout 300 python tools/lat.py "instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" "instances=1 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1" > gpurun_out/r2v1_lat.jsonl 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2v1_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --inplace-steps 0 --sweep "" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/r2v1_prof python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --inplace-steps 0 --sweep "" > gpurun_out/r2v1_ncu.log 2>&1
ncu -i gpurun_out/r2v1_prof.ncu-rep --page raw --csv > gpurun_out/r2v1_prof_raw.csv 2>/dev/null
ncu -i gpurun_out/r2v1_prof.ncu-rep --page details --csv > gpurun_out/r2v1_prof_details.csv 2>/dev/null
rm -f gpurun_out/r2v1_prof.ncu-rep
tail -3 gpurun_out/r2v1_pytest_new.log gpurun_out/r2v1_pytest_all.log; cat gpurun_out/r2v1_bench.json gpurun_out/r2v1_lat.jsonl
