#!/bin/bash
# A/B of library builds on the C5 bench step: scratch/ab_bench.sh tag1 tag2 ... (tree = in-tree build)
for v in "$@"; do
  if [ "$v" = tree ]; then unset AGNN_LIB; else export AGNN_LIB=scratch/libagnn_$v.so; fi
  python bench.py --no-cpu-baseline --no-bf16-line --no-e2e --steps 5 --warmup 3 ${BENCH_ARGS} > gpurun_out/ab_$v.json 2> gpurun_out/ab_$v.err
  python scratch/bline.py gpurun_out/ab_$v.json
done
