# HEAD at the end of round 2: smoke, the whole GPU suite, the bench line, the launch list and an ncu capture of the bench kernel
# an ncu --set full capture of the bench kernel
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final3.log 2>&1; echo "smoke=$?" >> gpurun_out/smoke_final3.log
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_final3.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_final3.log
python bench.py > gpurun_out/bench_final3.json 2> gpurun_out/bench_final3.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_final3.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_final3 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_final3.log 2>&1
ncu -i gpurun_out/prof_ring_ar8_final3.ncu-rep --page raw --csv > gpurun_out/prof_final3_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_ring_ar8_final3.ncu-rep --page details --csv > gpurun_out/prof_final3_details.csv 2>/dev/null
rm -f gpurun_out/prof_ring_ar8_final3.ncu-rep
tail -n 3 gpurun_out/smoke_final3.log gpurun_out/pytest_gpu_final3.log; head -c 1200 gpurun_out/bench_final3.json
