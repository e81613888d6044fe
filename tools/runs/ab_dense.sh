for i in 1 2; do
(cd _old && python bench.py --T 8 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed 's/^{/{"variant": "old", /') >> gpurun_out/ab_dense.jsonl
FFTSTENCIL_ALGO=dense python bench.py --T 8 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed 's/^{/{"variant": "new", /' >> gpurun_out/ab_dense.jsonl
done
