#!/bin/bash
# Source-level counters (instructions per SASS line, warp-state samples, pipe
# utilisation) of one compress or decompress launch at config 5; fewer sections than
# --set full, so the application replay of the 96 GiB working set stays short.
# usage: scripts/ncu_src_cfg5.sh <lib.so> <tag> [kernel regex] [cfg]
LIB=$1; TAG=$2; K=${3:-^compress_kernel}; CFG=${4:-cfg5}
mkdir -p gpurun_out
CSZP2_LIB=$LIB timeout -s KILL 1200 ncu --section SourceCounters --section WarpStateStats --section SchedulerStats \
  --section ComputeWorkloadAnalysis --section InstructionStats --section LaunchStats --section Occupancy \
  --replay-mode application --clock-control none --import-source on \
  --kernel-name-base function -k regex:"$K" -s 1 -c 1 -o gpurun_out/src_$TAG -f \
  python scripts/prof_one.py $CFG outlier 2 > gpurun_out/ncu_src_$TAG.log 2>&1
echo "ncu rc=$? $(tail -2 gpurun_out/ncu_src_$TAG.log)"
