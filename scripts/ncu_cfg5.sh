#!/bin/bash
# ncu --set full of one compress launch at config 5 (application replay: the 96 GiB of
# buffers cannot be saved/restored per pass). usage: scripts/ncu_cfg5.sh <lib.so> <tag> [cfg]
LIB=$1; TAG=$2; CFG=${3:-cfg5}
mkdir -p gpurun_out
CSZP2_LIB=$LIB timeout -s KILL 1500 ncu --set full --replay-mode application --clock-control none --import-source on \
  --kernel-name-base function -k regex:"^compress_kernel" -s 1 -c 1 -o gpurun_out/prof_$TAG -f \
  python scripts/prof_one.py $CFG outlier 2 > gpurun_out/ncu_$TAG.log 2>&1
echo "ncu rc=$? $(tail -2 gpurun_out/ncu_$TAG.log)"
