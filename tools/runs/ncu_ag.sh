mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
ncu --set full --clock-control none --import-source on -k regex:resccl -s 2 -c 1 -o gpurun_out/ag1 python tools/one_ag.py 1 allgather > gpurun_out/ncu_ag1.log 2>&1
ncu -i gpurun_out/ag1.ncu-rep --page source --csv --print-source sass > gpurun_out/ag1_sass.csv 2>/dev/null
ncu -i gpurun_out/ag1.ncu-rep --page details --csv > gpurun_out/ag1_details.csv 2>/dev/null
ncu --set full --clock-control none --import-source on -k regex:resccl -s 2 -c 1 -o gpurun_out/rs1 python tools/one_ag.py 1 reducescatter > gpurun_out/ncu_rs1.log 2>&1
ncu -i gpurun_out/rs1.ncu-rep --page source --csv --print-source sass > gpurun_out/rs1_sass.csv 2>/dev/null
ncu -i gpurun_out/rs1.ncu-rep --page details --csv > gpurun_out/rs1_details.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
ls -la gpurun_out/ag1_sass.csv gpurun_out/rs1_sass.csv; tail -3 gpurun_out/ncu_ag1.log
