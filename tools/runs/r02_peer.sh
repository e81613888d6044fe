# peer-memory transport: multi-process GPU tests (processes share the box's GPU), then the
# rest of the dist tests
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
nvidia-smi -L
timeout 1200 python -m pytest -q -x -m gpu tests/test_gpu_dist.py -k peer 2>&1 | tail -15
timeout 600 python -m pytest -q -m gpu tests/test_gpu_dist.py 2>&1 | tail -2
