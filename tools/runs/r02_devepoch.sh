mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
R="instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"
for de in 1 0; do
PHASE_NOGRAPH=1 PHASE_RAW=gpurun_out/phase_raw_de$de.jsonl PHASE_OPTS="$R devepoch=$de" timeout 300 python tools/phase_trace.py 16777216 > gpurun_out/phase_de$de.jsonl 2>&1
done
