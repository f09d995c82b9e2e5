mkdir -p gpurun_out
cat > /tmp/ttv_run.py <<'PY'
import torch, sys
sys.path.insert(0, ".")
import paper_conf_iiswc_lilwlob20_b200 as pasta, synth_inputs as si
cfg = si.CONFIGS["h"]
x = pasta.pasta_gen_powerlaw(cfg["dims"], cfg["nnz"], cfg["seed"], kind=1)
MF = pasta.pasta_coo_fibers(x, 0)
v = torch.rand(cfg["dims"][0], device="cuda"); y = torch.empty(MF, device="cuda")
for _ in range(5): pasta.pasta_ttv_coo(x, 0, v, out=y)
torch.cuda.synchronize()
PY
timeout 900 ncu --set full --clock-control none -k regex:ttv_segsum -s 3 -c 1 -o /tmp/ttv python /tmp/ttv_run.py > gpurun_out/ttv.log 2>&1
python tools/ncu_summary.py full /tmp/ttv.ncu-rep h_ttv gpurun_out/ncu_ttv.md ttv > /dev/null
