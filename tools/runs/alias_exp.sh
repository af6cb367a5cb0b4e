export RESCCL_TIMEOUT_MS=20000
for o in "instances=36 nwarps=8 tmastages=3 tmatile=8192" \
         "instances=36 nwarps=8 tmastages=6 tmatile=8192 smemalias=1" \
         "instances=36 nwarps=8 tmastages=4 tmatile=12288 smemalias=1" \
         "instances=18 nwarps=16 tmastages=8 tmatile=12288 smemalias=1" \
         "instances=18 nwarps=16 tmastages=6 tmatile=16384 smemalias=1"; do
  echo "== $o" >> gpurun_out/alias_exp.txt
  PHASE_OPTS="$o chunkbytes=16777216 fifodepth=2 direct=1" timeout 300 python tools/phases.py 2>&1 | head -3 >> gpurun_out/alias_exp.txt
done
