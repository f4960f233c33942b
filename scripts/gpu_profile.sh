#!/bin/bash
# Run on the GPU box (via gpurun): bench line, ncu launch list, ncu --set full captures.
# usage: scripts/gpu_profile.sh <tag> [bench|list|full|all]
set -u
TAG=${1:-r01}; WHAT=${2:-all}
OUT=gpurun_out
mkdir -p $OUT
echo "host: $(nproc) cores, $(free -g | awk '/Mem/{print $2}') GiB RAM"
if [[ $WHAT == bench || $WHAT == all ]]; then
  timeout -s KILL 900 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
  tail -c 4000 $OUT/bench_$TAG.json; tail -3 $OUT/bench_$TAG.err
fi
if [[ $WHAT == list || $WHAT == all ]]; then
  # launch list of the bench command (our kernels only; cold-cache, serialised)
  timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
      --kernel-name-base function -k regex:"compress_kernel|decompress_kernel|minmax_kernel|container_index" -c 30 --csv \
      --log-file $OUT/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-plain --e2e-steps 1 \
      --cpu-sample-log2 16 > $OUT/ncu_list_$TAG.log 2>&1; echo "ncu list rc=$?"
fi
if [[ $WHAT == full || $WHAT == all ]]; then
  # --set full of each kernel on config 3b (512 MiB; replaying config 5's 96 GiB of buffers is impractical)
  for K in compress_kernel decompress_kernel minmax_kernel; do
    timeout -s KILL 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:"^$K" -s 3 -c 1 \
        -o $OUT/prof_${K}_$TAG -f python bench.py --config cfg3b --steps 1 --warmup 3 --no-plain --e2e-steps 1 \
        --cpu-sample-log2 16 > $OUT/ncu_full_${K}_$TAG.log 2>&1; echo "ncu full $K rc=$?"
  done
fi
