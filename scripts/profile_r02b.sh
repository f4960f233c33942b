#!/bin/bash
# Round-2 second-session profiling pass on the GPU box: ncu launch list (duration + DRAM
# bytes per launch) of the bench command, the same for the nD kernels on configs 2/3b/4b,
# and the Table VI analog. usage: scripts/profile_r02b.sh <tag>
TAG=${1:-r02b}
OUT=gpurun_out
mkdir -p $OUT
timeout -s KILL 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --kernel-name-base function -k regex:"compress_kernel|decompress_kernel|minmax_kernel|container_index|zero_scratch" --csv \
    --log-file $OUT/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --config-steps 3 --e2e-steps 1 \
    --cpu-sample-log2 16 > $OUT/ncu_list_$TAG.log 2>&1; echo "ncu list rc=$?"
python scripts/launch_summary.py $OUT/launches_$TAG.csv $OUT/${TAG}_launches.md "launch list, bench.py, $TAG"
for c in cfg2 cfg3b cfg4b; do
  timeout -s KILL 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
      --kernel-name-base function -k regex:"_nd_|minmax" --csv --log-file $OUT/nd_launches_${c}_$TAG.csv \
      python scripts/prof_nd.py $c outlier 2 > /dev/null 2>&1; echo "ncu nd $c rc=$?"
done
# one process per config: after config 2 in the same process, config 3a's 3D decompression
# measures 0.43-0.49 instead of 0.66 (not understood)
for c in cfg2 cfg3a cfg3b cfg4b; do
  timeout -s KILL 150 python scripts/nd_table.py $c 2>> $OUT/nd_table_$TAG.err
done > $OUT/nd_table_$TAG.jsonl
echo "nd_table rc=$?"
