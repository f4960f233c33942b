#!/bin/bash
# Source counters of one nD kernel launch (compress_nd_kernel / decompress_nd_kernel).
# usage: scripts/ncu_src_nd.sh <tag> <kernel regex> <cfg> <enc>
TAG=$1; K=${2:-^compress_nd_kernel}; CFG=${3:-cfg3b}; ENC=${4:-outlier}
mkdir -p gpurun_out
timeout -s KILL 900 ncu --section SourceCounters --section WarpStateStats --section SchedulerStats \
  --section ComputeWorkloadAnalysis --section InstructionStats --section LaunchStats --section Occupancy \
  --section MemoryWorkloadAnalysis --section SpeedOfLight \
  --clock-control none --import-source on \
  --kernel-name-base function -k regex:"$K" -s 2 -c 1 -o gpurun_out/src_$TAG -f \
  python scripts/prof_nd.py $CFG $ENC 3 > gpurun_out/ncu_src_$TAG.log 2>&1
echo "ncu $TAG rc=$? $(tail -1 gpurun_out/ncu_src_$TAG.log)"
