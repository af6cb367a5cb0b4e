# source-level ncu capture of ring AllReduce at 16 MiB per rank (mid-size: where a hop's fixed cost shows)
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
python tools/one_coll.py allreduce 16 "instances=14 nwarps=8 chunkbytes=33554432 direct=1" 4 > gpurun_out/one16.log 2>&1 && \
ncu --set full --clock-control none --import-source on -k regex:resccl -s 3 -c 1 -o gpurun_out/prof_ring16 python tools/one_coll.py allreduce 16 "instances=14 nwarps=8 chunkbytes=33554432 direct=1" 4 > gpurun_out/ncu16.log 2>&1
ls -la gpurun_out; tail -3 gpurun_out/ncu16.log
