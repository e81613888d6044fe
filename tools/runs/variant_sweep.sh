#!/bin/bash
# Fused 2D kernel variant ablation: parity first, then bench lines per (variant, workload, T).
out=${1:-gpurun_out/variants.jsonl}
: > $out
for V in 0 1 2; do
  FFTSTENCIL_VARIANT=$V python -m pytest tests/test_gpu_parity.py -q -x -k "parity_vs_oracle or T_invariance or aliasing or semigroup" 2>&1 | tail -1 | sed "s/^/V=$V parity: /"
done
for V in 0 1 2; do
  for cfg in "heat2d 4" "heat2d 8" "heat2d 16" "box2d49p 3" "box2d49p 4"; do
    set -- $cfg
    FFTSTENCIL_VARIANT=$V python bench.py --workload $1 --T $2 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": $V, /" >> $out
  done
done
