# NEXT-3: Fig. 7-style ablation ladder on B200 (Heat-2D 10240^2, 1000 steps, own kernels only)
out=${1:-gpurun_out/ablation.jsonl}
: > $out
run() { tag=$1; shift; env "$@" python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline ${BENCH_ARGS} | tail -1 | sed "s/^{/{\"variant\": \"$tag\", /" >> $out; }
BENCH_ARGS="--T 1" run "A unfused-3-kernels-T1" FFTSTENCIL_ALGO=unfused
BENCH_ARGS="--T 1" run "B fused-dense-T1" FFTSTENCIL_ALGO=dense
BENCH_ARGS="" run "C fused-dense-Tauto" FFTSTENCIL_ALGO=dense
BENCH_ARGS="" run "C' unfused-Tauto" FFTSTENCIL_ALGO=unfused
BENCH_ARGS="" run "D factored-cpasync-Tauto" FFTSTENCIL_ALGO=factored FFTSTENCIL_TMA=0
BENCH_ARGS="" run "E factored-tma-Tauto" FFTSTENCIL_ALGO=factored
