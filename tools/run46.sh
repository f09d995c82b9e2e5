mkdir -p gpurun_out
rm -f gpurun_out/sweep21.txt
python - >> gpurun_out/sweep21.txt <<'PY'
import torch
p = torch.cuda.get_device_properties(0)
print("L2", p.L2_cache_size, "persist max", getattr(p, "persisting_l2_cache_max_size", None))
PY
for MB in 16 24 32 40; do
  echo "== h PERSIST=1 HOT_MB=$MB" >> gpurun_out/sweep21.txt
  PASTA_HOT_PERSIST=1 PASTA_HOT_MB=$MB timeout 900 python tools/sweep.py --config h --variants 0 --runs 0,128 --formats coo --reps 10 >> gpurun_out/sweep21.txt 2>&1
done
for MB in 24 32 48 64; do
  echo "== c3 PERSIST=1 HOT_MB=$MB" >> gpurun_out/sweep21.txt
  PASTA_HOT_PERSIST=1 PASTA_HOT_MB=$MB timeout 900 python tools/sweep.py --config c3 --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep21.txt 2>&1
done
for MB in 32 64; do
  echo "== c5 PERSIST=1 HOT_MB=$MB" >> gpurun_out/sweep21.txt
  PASTA_HOT_PERSIST=1 PASTA_HOT_MB=$MB timeout 900 python tools/sweep.py --config c5 --variants 0 --runs 0 --formats coo --reps 3 >> gpurun_out/sweep21.txt 2>&1
done
