# round-2 closing evidence after making the 3D band concurrent (side stream): smoke, GPU tests,
# launch list, ncu of the band kernel, multi-process peer worker log
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -4 | tee gpurun_out/r02j_smoke.txt
timeout 2400 python -m pytest tests -q -m gpu 2>&1 | tail -4 | tee gpurun_out/r02j_gpu_tests.txt
( time timeout 900 python bench.py > gpurun_out/r02j_bench.jsonl 2> gpurun_out/r02j_bench.err ) 2>&1 | tail -3
( time timeout 600 python bench.py --impl reference > gpurun_out/r02j_reference.jsonl ) 2>&1 | tail -3
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02j_launches.csv python bench.py --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:band_cone -s 3 -c 1 -o gpurun_out/r02j_band3d python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncuband rc=$?
FFTSTENCIL_PEER_FUSED=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node=3 --master-addr=127.0.0.1 --master-port=29551 tests/_peer_worker.py 2>&1 | grep case > gpurun_out/r02j_peer_worker.txt
FFTSTENCIL_BENCH_SHARE_GPU=1 timeout 900 python bench.py --gpus 2 --steps 2 --warmup 1 --no-e2e > gpurun_out/r02j_bench_n2_shared.jsonl 2>/dev/null; echo n2 rc=$?
