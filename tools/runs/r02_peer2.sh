# peer transport after adding the connect-time probe: multi-process tests + the N = 2 bench path (shared GPU)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest -q -m gpu tests/test_gpu_dist.py 2>&1 | tail -2
FFTSTENCIL_BENCH_SHARE_GPU=1 timeout 900 python bench.py --gpus 2 --steps 2 --warmup 1 --workload box2d9p_weak --no-e2e 2>/dev/null | tail -1 | head -c 400; echo
