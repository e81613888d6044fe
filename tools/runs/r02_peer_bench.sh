# the N > 1 bench path end to end on a one-GPU box: two ranks share device 0 over the peer
# transport (a harness test, not a scaling number), 2D and 3D weak slabs; then N = 1 of the same slab
FFTSTENCIL_BENCH_SHARE_GPU=1 timeout 900 python bench.py --gpus 2 --steps 2 --warmup 1 --workload heat3d_weak > gpurun_out/r02_peer_bench3d.jsonl 2> gpurun_out/r02_peer_bench3d.err; echo rc=$?
FFTSTENCIL_BENCH_SHARE_GPU=1 timeout 900 python bench.py --gpus 2 --steps 2 --warmup 1 --workload box2d9p_weak > gpurun_out/r02_peer_bench2d.jsonl 2> gpurun_out/r02_peer_bench2d.err; echo rc=$?
timeout 900 python bench.py --steps 2 --warmup 1 --workload heat3d_weak --no-per-config --no-cpu-baseline > gpurun_out/r02_peer_bench3d_n1.jsonl 2>/dev/null; echo rc=$?
for f in gpurun_out/r02_peer_bench3d.jsonl gpurun_out/r02_peer_bench2d.jsonl gpurun_out/r02_peer_bench3d_n1.jsonl; do
  python -c "import json;d=json.loads(open('$f').read().strip().splitlines()[-1]);print('$f', d['n_gpus'], round(d['value'],1), d['ms_per_step'], d['config'].get('transport'), d.get('shared_gpu','')[:20], (d.get('e2e') or {}).get('value'))"
done
tail -3 gpurun_out/r02_peer_bench3d.err
