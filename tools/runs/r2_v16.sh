# r02: ncu of the bench kernel at the r02 defaults (launch list + full set), and the mesh kernel
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2v16_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --inplace-steps 0 --sweep "" --tuned-sweep "" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/r2v16_prof python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --inplace-steps 0 --sweep "" --tuned-sweep "" > gpurun_out/r2v16_ncu.log 2>&1
ncu -i gpurun_out/r2v16_prof.ncu-rep --page raw --csv > gpurun_out/r2v16_prof_raw.csv 2>/dev/null
ncu -i gpurun_out/r2v16_prof.ncu-rep --page details --csv > gpurun_out/r2v16_prof_details.csv 2>/dev/null
rm -f gpurun_out/r2v16_prof.ncu-rep
ncu --set full --clock-control none -k regex:resccl -s 3 -c 1 -o gpurun_out/r2v16_mesh python tools/one_coll.py allreduce 256 "instances=14 chunkbytes=8388608 linkmodel=port nwarps=8 fifodepth=2 direct=1" 5 hm "g=8" > gpurun_out/r2v16_ncu_mesh.log 2>&1
ncu -i gpurun_out/r2v16_mesh.ncu-rep --page raw --csv > gpurun_out/r2v16_mesh_raw.csv 2>/dev/null
rm -f gpurun_out/r2v16_mesh.ncu-rep
grep -c resccl gpurun_out/r2v16_launches.csv; tail -2 gpurun_out/r2v16_ncu.log
