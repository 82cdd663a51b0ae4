#!/bin/bash
# dev experiment: which part of the split-K epilogue costs time
for shape in "256 5120 5120" "8 20480 5120"; do
  for S in 1 8; do
    for D in 0 1 2 4 3 7; do
      echo -n "shape=$shape S=$S dbg=$D : "
      LIGER_GEMM_FORCE_SPLITS=$S LIGER_GEMM_DBG=$D python tools/split_sweep.py child $shape | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(round(d['us'],1))"
    done
  done
done
