# HEAD evidence refresh: Table 3 analogue at the best geometries, the C5 analogue, and ncu captures of the
# size-tuned classes (2x4 at 4 MiB, port-model mesh at 16 MiB)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=30000
timeout 900 python tools/tb_util.py 256 best > gpurun_out/tb_util_head.jsonl 2>&1
timeout 900 python tools/overlap.py > gpurun_out/overlap_head.jsonl 2>&1
python tools/one_coll.py allreduce 4 "instances=4 nwarps=8 chunkbytes=524288 direct=1" 4 hm g=4 > gpurun_out/one4.log 2>&1 && \
ncu --set full --clock-control none -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_hm4_4MiB python tools/one_coll.py allreduce 4 "instances=4 nwarps=8 chunkbytes=524288 direct=1" 4 hm g=4 > gpurun_out/ncu_hm4.log 2>&1
ncu -i gpurun_out/prof_hm4_4MiB.ncu-rep --page raw --csv > gpurun_out/prof_hm4_4MiB_raw.csv 2>/dev/null
ncu --set full --clock-control none -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_mesh_16MiB python tools/one_coll.py allreduce 16 "instances=18 nwarps=8 linkmodel=port chunkbytes=8388608 direct=1" 4 hm g=8 > gpurun_out/ncu_mesh16.log 2>&1
ncu -i gpurun_out/prof_mesh_16MiB.ncu-rep --page raw --csv > gpurun_out/prof_mesh_16MiB_raw.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
head -c 1500 gpurun_out/tb_util_head.jsonl; tail -3 gpurun_out/overlap_head.jsonl
