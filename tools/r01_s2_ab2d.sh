# A/B of 2D radix-engine tuning builds (one box, back to back)
for lib in "" __DBF_TW_POW_1 __DBF_TW_POW_2 __DBF_UNROLL_2 __DBF_TW_POW_2_DBF_UNROLL_2; do
  so=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil$lib.so
  for w in heat2d box2d49p; do
    FFTSTENCIL_LIB=$PWD/$so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/ab_$w$lib.jsonl 2>&1
    python - "$lib" "$w" gpurun_out/ab_$w$lib.jsonl <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[3]).read().strip().splitlines()[-1])
    print(f"{sys.argv[1] or 'default':32s} {sys.argv[2]:10s} {d['value']:8.1f} GSt/s fused {d['roofline']['fused_ms_avg']:.4f} ms frac {d['roofline']['frac']:.3f}")
except Exception as e:
    print(sys.argv[1], sys.argv[2], "FAILED", e)
PY
  done
done
FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DBF_TW_POW_2.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d_engines or full_size_sampled" 2>&1 | tail -3
