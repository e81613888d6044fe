python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or 3d or periodic or full_size" 2>&1 | tail -1
FFTSTENCIL_TMA=0 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle" 2>&1 | tail -1
rm -f gpurun_out/r01_run10.jsonl
for w in heat2d box2d49p heat3d; do python bench.py --workload $w --steps 2 --warmup 2 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run10.jsonl; done
ncu --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,gpu__time_duration.sum -k regex:fft -s 2 -c 1 --csv python bench.py --steps 1 --warmup 1 --time-steps 33 --no-e2e --no-cpu-baseline 2>&1 | grep -E "conflicts|wavefronts|duration" | cut -c1-300
