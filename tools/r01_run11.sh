python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "unfused or parity_vs_oracle" 2>&1 | tail -1
bash tools/ablation.sh gpurun_out/r01_ablation.jsonl
