mkdir -p gpurun_out
cat > /tmp/pp.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch, gen, paper_conf_sc_dastgeerlk12_b200 as pepp
n = 31_622_777
A = gen.uniform(n, n, 16, seed=100 + n % 97)
x = torch.from_numpy(gen.vector(7, gen.REAL, n)).cuda(); y = torch.empty(n, dtype=torch.float64, device="cuda")
plan = pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_PANEL)
for _ in range(2): plan.exec(x, y, force=pepp.Choice(pepp.V_PANEL, 22))
torch.cuda.synchronize()
PY
timeout 900 ncu --set full --clock-control none -k regex:panel_kernel -s 10 -c 1 -o gpurun_out/r2_panel -f python /tmp/pp.py > gpurun_out/r2_panel.log 2>&1; echo rc=$?
python tools/ncu_summary.py gpurun_out/r2_panel.ncu-rep
ncu -i gpurun_out/r2_panel.ncu-rep --page raw --csv 2>/dev/null | python -c "
import csv,sys
r=list(csv.reader(sys.stdin)); h=r[0]; v=r[-1]
d={a:b for a,b in zip(h,v)}
st=sorted(((k,float(d[k])) for k in d if k.startswith('smsp__pcsamp_warps_issue_stalled_') and not k.endswith('not_issued') and d[k].replace('.','').isdigit()), key=lambda t:-t[1])
tot=sum(x for _,x in st) or 1
for k,x in st[:8]: print(f'{x/tot*100:6.1f}%  {k}')
for k in ['dram__throughput.avg.pct_of_peak_sustained_elapsed','lts__t_sector_hit_rate.pct','launch__grid_size','lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum','lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum']:
    print(k, d.get(k))
"
