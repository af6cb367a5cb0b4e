# HEAD (device epochs, 32 KiB TMA slices, host-buffer staging): gpu suite, bench line, launch list + ncu --set full of the bench kernel
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_v14.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v14.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_v14.log
python bench.py > gpurun_out/bench_v14.json 2> gpurun_out/bench_v14.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v14.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_v14 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_v14.log 2>&1
ncu -i gpurun_out/prof_ring_ar8_v14.ncu-rep --page raw --csv > gpurun_out/prof_v14_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_ring_ar8_v14.ncu-rep --page details --csv > gpurun_out/prof_v14_details.csv 2>/dev/null
rm -f gpurun_out/prof_ring_ar8_v14.ncu-rep
tail -3 gpurun_out/pytest_gpu_v14.log; cat gpurun_out/bench_v14.json
