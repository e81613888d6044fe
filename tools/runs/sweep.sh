#!/bin/bash
# Run bench.py over the BASELINE configurations (and the 2D T sweep); one JSON line each.
out=${1:-gpurun_out/sweep.jsonl}
: > $out
for T in 1 2 4 8 12 16; do python bench.py --workload heat2d --T $T --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> $out; done
for T in 1 2 4 8 12 16; do python bench.py --workload box2d9p --T $T --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> $out; done
for w in star2d13p box2d49p; do for T in 0 2 3 4; do python bench.py --workload $w --T $T --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> $out; done; done
for w in heat3d box3d27p; do for T in 0 1 2 3; do python bench.py --workload $w --T $T --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> $out; done; done
python bench.py --workload heat1d --T 8 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline | tail -1 >> $out
