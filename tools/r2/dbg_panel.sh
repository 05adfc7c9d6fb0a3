cat > /tmp/pp2.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch, gen, paper_conf_sc_dastgeerlk12_b200 as pepp
n = 31_622_777
A = gen.uniform(n, n, 16, seed=100 + n % 97)
x = torch.from_numpy(gen.vector(7, gen.REAL, n)).cuda(); y = torch.empty(n, dtype=torch.float64, device="cuda")
plan = pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_PANEL)
print([c.name for c in plan.candidates()])
for _ in range(2): print(plan.exec(x, y, force=pepp.Choice(pepp.V_PANEL, 22)))
torch.cuda.synchronize()
PY
python /tmp/pp2.py
