#!/bin/bash
# compute-sanitizer passes (memcheck, racecheck, synccheck, initcheck) over smoke() and the
# small-size GPU parity tests. Run on the GPU box: bash scripts/sanitize.sh <tag>
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
CS=/usr/local/cuda/bin/compute-sanitizer
SEL='test_small_sizes_rel or test_special_fields or test_decompress_rejects_corrupt_streams or test_random_access_ranges or test_decompress_tilewise_ablation or test_incompressible_many_tiles or test_nd_parity_rel'
for TOOL in memcheck racecheck synccheck initcheck; do
  echo "== $TOOL smoke" >> $OUT/sanitize_$TAG.txt
  timeout 240 $CS --tool $TOOL --error-exitcode 99 python -c "import __graft_entry__ as g; g.smoke()" \
      2>&1 | tail -4 >> $OUT/sanitize_$TAG.txt; echo "rc=${PIPESTATUS[0]}" >> $OUT/sanitize_$TAG.txt
done
for TOOL in memcheck racecheck synccheck; do
  echo "== $TOOL pytest ($SEL)" >> $OUT/sanitize_$TAG.txt
  timeout 420 $CS --tool $TOOL --error-exitcode 99 python -m pytest tests/test_gpu_parity.py tests/test_gpu_nd.py -m gpu -q -x \
      -k "$SEL or small" -p no:cacheprovider 2>&1 | tail -4 >> $OUT/sanitize_$TAG.txt; echo "rc=${PIPESTATUS[0]}" >> $OUT/sanitize_$TAG.txt
done
cat $OUT/sanitize_$TAG.txt
