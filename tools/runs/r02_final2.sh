# HEAD after the early loop exit: smoke, the whole GPU suite, the bench line, the launch list and an ncu --set full capture of the bench kernel
# an ncu --set full capture of the bench kernel
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final2.log 2>&1; echo "smoke=$?" >> gpurun_out/smoke_final2.log
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_final2.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_final2.log
python bench.py > gpurun_out/bench_final2.json 2> gpurun_out/bench_final2.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_final2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring_ar8_final2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full_final2.log 2>&1
ncu -i gpurun_out/prof_ring_ar8_final2.ncu-rep --page raw --csv > gpurun_out/prof_final2_raw.csv 2>/dev/null
ncu -i gpurun_out/prof_ring_ar8_final2.ncu-rep --page details --csv > gpurun_out/prof_final2_details.csv 2>/dev/null
rm -f gpurun_out/prof_ring_ar8_final2.ncu-rep
tail -n 3 gpurun_out/smoke_final2.log gpurun_out/pytest_gpu_final2.log; head -c 1200 gpurun_out/bench_final2.json
