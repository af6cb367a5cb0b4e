mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/tmamin.jsonl
: > $O
for tm in 163840 65536 32768 16384; do
CS_SIZES=2,4,16,64 CS_CHUNKS=32768 CS_OPTS="tmamin=$tm nwarps=8 tmastages=2 tmatile=24576" timeout 300 python tools/chunk_sweep.py >> $O 2>&1
done
cat $O
