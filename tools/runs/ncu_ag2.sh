mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
ncu --set full --clock-control none --import-source on -k regex:resccl -s 2 -c 1 -o gpurun_out/ag2 python tools/one_ag.py 1 allgather > gpurun_out/ncu_ag2.log 2>&1
ncu -i gpurun_out/ag2.ncu-rep --page source --csv --print-source sass > gpurun_out/ag2_sass.csv 2>/dev/null
ncu -i gpurun_out/ag2.ncu-rep --page raw --csv > gpurun_out/ag2_raw.csv 2>/dev/null
ncu --set full --clock-control none --import-source on -k regex:resccl -s 2 -c 1 -o gpurun_out/ar2 python tools/one_ag.py 1 allreduce > gpurun_out/ncu_ar2.log 2>&1
ncu -i gpurun_out/ar2.ncu-rep --page source --csv --print-source sass > gpurun_out/ar2_sass.csv 2>/dev/null
ncu -i gpurun_out/ar2.ncu-rep --page raw --csv > gpurun_out/ar2_raw.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
