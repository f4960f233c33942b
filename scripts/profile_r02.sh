#!/bin/bash
# Round-2 profiling pass on the GPU box: launch list of the bench command, ncu --set full
# traffic per (config, mode, kernel), source counters of the cfg4a Plain compressor.
# usage: scripts/profile_r02.sh <tag>
TAG=${1:-r02}
OUT=gpurun_out
mkdir -p $OUT
timeout -s KILL 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --kernel-name-base function -k regex:"compress_kernel|decompress_kernel|minmax_kernel|container_index|zero_scratch" --csv \
    --log-file $OUT/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --config-steps 3 --e2e-steps 1 \
    --cpu-sample-log2 16 > $OUT/ncu_list_$TAG.log 2>&1; echo "ncu list rc=$?"
timeout -s KILL 1500 python scripts/ncu_traffic.py $OUT/ncu_traffic_$TAG.json cfg1:plain cfg1:outlier cfg2:plain cfg2:outlier \
    cfg3a:plain cfg3a:outlier cfg3b:plain cfg3b:outlier cfg4a:plain cfg4a:outlier cfg4b:plain cfg4b:outlier \
    > $OUT/ncu_traffic_$TAG.log 2>&1; echo "ncu traffic rc=$?"
scripts/ncu_src.sh c4aP_$TAG ^compress_kernel cfg4a plain
scripts/ncu_src.sh c4aO_$TAG ^compress_kernel cfg4a outlier
