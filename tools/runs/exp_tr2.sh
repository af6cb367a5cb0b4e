mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
G="nwarps=16 tmastages=4 tmatile=12288 chunkbytes=33554432 fifodepth=2 direct=1 trace=2"
timeout 120 python tools/exp_ag.py reducescatter 8 256 0 "instances=4 $G" > gpurun_out/tr2_rs.txt 2>&1
timeout 120 python tools/exp_ag.py allgather 8 256 0 "instances=4 $G" > gpurun_out/tr2_ag.txt 2>&1
tail -5 gpurun_out/tr2_rs.txt; tail -5 gpurun_out/tr2_ag.txt
