# r02: Table 3 analogue at each schedule's best geometry; ncu of DBT / HM / synth kernels; C3 budget sweep
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 600 python tools/tb_util.py 256 best > gpurun_out/r2v8_tbutil_best.jsonl 2> gpurun_out/r2v8_tbutil.err
timeout 600 python tools/tb_util.py 64 r01 > gpurun_out/r2v8_tbutil_r01.jsonl 2>> gpurun_out/r2v8_tbutil.err
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__block_size,launch__registers_per_thread,sm__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,smsp__sass_inst_executed_op_local_ld.sum"
for c in "allreduce dbt '' instances=6_chunkbytes=8388608_nwarps=8_direct=1" "allreduce hm g=4 instances=4_chunkbytes=1048576_nwarps=8_direct=1" "allgather synth seed=0_fanout=2 instances=4_chunkbytes=8388608_nwarps=8_direct=1" "reducescatter synth seed=0_fanout=2 instances=4_chunkbytes=1048576_nwarps=8_direct=1"; do
  set -- $c; coll=$1; algo=$2; g=$(echo $3 | tr '_' ' ' | tr -d "'"); o=$(echo $4 | tr '_' ' ')
  timeout 600 ncu --metrics $M --clock-control none -k regex:resccl -s 3 -c 1 --csv python tools/one_coll.py $coll 256 "$o" 5 $algo "$g" > gpurun_out/r2v8_ncu_${algo}_${coll}.csv 2> gpurun_out/r2v8_ncu_${algo}_${coll}.err
done
timeout 900 python tools/sweep.py c3 > gpurun_out/r2v8_c3.jsonl 2> gpurun_out/r2v8_c3.err
cat gpurun_out/r2v8_tbutil_best.jsonl; grep -h "gpu__time_duration\|dram__bytes" gpurun_out/r2v8_ncu_*.csv | cut -c1-300
