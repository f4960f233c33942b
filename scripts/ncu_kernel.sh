#!/bin/bash
# ncu --set full (kernel replay) of one launch of a kernel on a config that fits replay.
# usage: scripts/ncu_kernel.sh <kernel-regex> <tag> [cfg] [enc]
K=$1; TAG=$2; CFG=${3:-cfg3b}; ENC=${4:-outlier}
mkdir -p gpurun_out
timeout -s KILL 900 ncu --set full --clock-control none --import-source on --kernel-name-base function \
  -k regex:"$K" -s 2 -c 1 -o gpurun_out/prof_$TAG -f python scripts/prof_one.py $CFG $ENC 3 > gpurun_out/ncu_$TAG.log 2>&1
echo "ncu $TAG rc=$? $(tail -1 gpurun_out/ncu_$TAG.log)"
