python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DB3_NG=2" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD2 FAILED
ls paper_conf_ppopp_hanlcbzyczcy25_b200/*.so
cat > /tmp/dbg3d.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_hanlcbzyczcy25_b200 as fs
from synth import workloads as wl
import oracle
ext, r, T, steps = (60, 50, 45), 1, 2, 2
w = wl.seeded_weights("star", 3, r); u0 = wl.grid(ext, 3)
ref = oracle.stencil_run(u0, w, r, steps)
for env in [{"FFTSTENCIL_MAX_CTAS": "1"}, {"FFTSTENCIL_MAX_CTAS": "1", "FFTSTENCIL_TMA": "0"}, {"FFTSTENCIL_MAX_CTAS": "2"}, {}]:
    os.environ.update(env)
    p = fs.Plan(ext, w, r, T); a = torch.from_numpy(u0).cuda(); b = torch.empty_like(a)
    p.run(a, b, steps); torch.cuda.synchronize()
    d = np.abs(b.cpu().numpy() - ref)
    bad = np.argwhere(d > 1e-9)
    print(env, "max err", d.max(), "bad cells", len(bad), flush=True)
    if len(bad):
        h, S = 2, 12
        tiles = set(tuple((c - h) // S) for c in bad)
        print("  bad tiles (t0,t1,t2):", sorted(tiles)[:20], "count", len(tiles))
        print("  first bad", bad[:5].tolist(), "got", b.cpu().numpy()[tuple(bad[0])], "ref", ref[tuple(bad[0])])
    for k in env: del os.environ[k]
PY
python /tmp/dbg3d.py
FFTSTENCIL_LIB=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DB3_NG_2.so python /tmp/dbg3d.py
for lib in libfftstencil.so libfftstencil__DB3_NG_2.so; do
  FFTSTENCIL_LIB=paper_conf_ppopp_hanlcbzyczcy25_b200/$lib timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config > gpurun_out/r02_3d_$lib.jsonl 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02_3d_$lib.jsonl').read().strip().splitlines()[-1]);print('$lib', round(d['value'],1), 'GSt/s', 'frac', round(d['roofline']['frac'],3), 'fused ms', round(d['roofline']['fused_ms_avg'],3))" || tail -5 gpurun_out/r02_3d_$lib.jsonl
done
