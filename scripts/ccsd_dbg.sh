cd $GRAFT_REPO_ROOT
for dbg in 0 1 2 4 3 5 6 7; do echo "== dbg $dbg"; EATSS_CCSD_TC_DBG=$dbg timeout 300 python scripts/time_kernel.py ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1; done
echo "== M48 dbg 2"; EATSS_CCSD_TC_DBG=2 timeout 300 python scripts/time_kernel.py ccsd_t_d1 48 1,1,1,48,1,48,48 --engine 2 --iters 5 2>&1 | tail -1
echo "== M48 dbg 6"; EATSS_CCSD_TC_DBG=6 timeout 300 python scripts/time_kernel.py ccsd_t_d1 48 1,1,1,48,1,48,48 --engine 2 --iters 5 2>&1 | tail -1
python - <<'PY'
import torch, time
x = torch.empty(12 * 1024**3 // 4, device="cuda"); y = torch.empty_like(x)
for _ in range(3): y.copy_(x)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize(); s.record()
for _ in range(5): y.copy_(x)
e.record(); torch.cuda.synchronize()
print("copy 12 GiB: %.2f TB/s" % (2 * x.numel() * 4 * 5 / (s.elapsed_time(e) * 1e-3) / 1e12))
PY
