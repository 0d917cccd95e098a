cd $GRAFT_REPO_ROOT
# dbg bits (development only): 1 no MMA, 2 no t3 traffic, 4 no v2 loads
for dbg in 0 1 2 4 5 6 7; do echo "== dbg $dbg"; EATSS_CCSD_TC_DBG=$dbg timeout 300 python scripts/time_kernel.py ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1; done
for xs in 3 4 5; do echo "== xstages $xs"; EATSS_CCSD_TC_XSTAGES=$xs timeout 300 python scripts/time_kernel.py ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1; done
echo "== order 0"; EATSS_CCSD_TC_ORDER=0 timeout 300 python scripts/time_kernel.py ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1
python - <<'PY'
import torch
x = torch.empty(48**6, device="cuda")
x.uniform_()
for _ in range(2): x.sub_(0.5)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize(); s.record()
for _ in range(5): x.sub_(0.5)
e.record(); torch.cuda.synchronize()
ms = s.elapsed_time(e) / 5
print("torch in-place RMW over t3 (48.9 GB): %.2f ms, %.2f TB/s" % (ms, 2 * x.numel() * 4 / ms / 1e9))
PY
timeout 900 python scripts/ccsd_variants.py
