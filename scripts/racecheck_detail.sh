#!/bin/bash
# racecheck with per-hazard detail (kernel, source lines) over smoke() and two parity tests
# usage: bash scripts/racecheck_detail.sh <tag>
TAG=${1:-r02}; OUT=gpurun_out; mkdir -p $OUT
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 600 $CS --tool racecheck --racecheck-report hazard --print-limit 400 python -m pytest tests/test_gpu_parity.py -m gpu -q -x \
    -k "test_small_sizes_rel and 100003 or test_incompressible_many_tiles and float32-outlier" -p no:cacheprovider > $OUT/race_$TAG.txt 2>&1
echo "rc=$?"
grep -E "^========= (Error|Warning)|kernels|\.cuh:" $OUT/race_$TAG.txt | sed 's/0x[0-9a-f]*//g' | sort | uniq -c | sort -rn | head -40
