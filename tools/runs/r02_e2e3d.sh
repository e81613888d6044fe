# Heat-3D e2e (pipelined run_host): pinned copy bandwidth and a Q / K sweep
python - <<'PY'
import torch, time
n = 1 << 27   # 1 GiB of float64
h = torch.empty(n, dtype=torch.float64).pin_memory(); d = torch.empty(n, dtype=torch.float64, device="cuda")
h2 = torch.empty(n, dtype=torch.float64).pin_memory(); d2 = torch.empty(n, dtype=torch.float64, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for _ in range(2): d.copy_(h, non_blocking=True); h.copy_(d, non_blocking=True)
torch.cuda.synchronize()
def t(f):
    torch.cuda.synchronize(); t0 = time.perf_counter(); f(); torch.cuda.synchronize(); return time.perf_counter() - t0
a = t(lambda: d.copy_(h, non_blocking=True)); b = t(lambda: h.copy_(d, non_blocking=True))
def both():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
c = t(both)
print(f"H2D {8*n/a/1e9:.1f} GB/s  D2H {8*n/b/1e9:.1f} GB/s  concurrent {8*n/c/1e9:.1f} GB/s each way")
PY
run() {  # K Q
  FFTSTENCIL_E2E_PIPE=$1 FFTSTENCIL_E2E_DEPTH=$2 timeout 600 python bench.py --workload heat3d --steps 3 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());e=d['e2e'];print('K=$1 Q=$2 device', round(d['value'],1), 'e2e', round(e['value'],1), 'e2e ms', round(e['ms_per_step'],1), 'dev ms', round(d['ms_per_step'],1))"
}
run 12 16; run 12 20; run 12 24; run 16 20; run 8 20; run 12 16
