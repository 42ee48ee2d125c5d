# k_update_pf with cp.async stages + static positions: parity, P sweep, ncu source view at P = 4.
python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_gputests.log 2>&1; tail -3 gpurun_out/t_gputests.log
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e"
for p in 1 4 16 64; do
  $B --partitions $p --refill 3 > gpurun_out/t_p${p}_rf3.json 2>/dev/null
  LT_LIBRARY=tools/variants/liblt_pf3.so $B --partitions $p --refill 3 > gpurun_out/t_p${p}_rf3_minb3.json 2>/dev/null
done
for f in gpurun_out/t_p*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1), s['sweeps'], s['update_launches'])"; done
ncu --set full --clock-control none --import-source on -k regex:k_update -s 20 -c 1 -f -o gpurun_out/t_pf_full \
  python tools/profile_run.py --partitions 4 --refill 3 --steps 2 > gpurun_out/t_pf_full.log 2>&1
python tools/ncu_summary.py report gpurun_out/t_pf_full.ncu-rep > gpurun_out/t_pf_full.txt 2>&1
ncu -i gpurun_out/t_pf_full.ncu-rep --page source --csv > gpurun_out/t_pf_full.src.csv 2>/dev/null
ncu -i gpurun_out/t_pf_full.ncu-rep --page raw --csv > gpurun_out/t_pf_full.raw.csv 2>/dev/null
rm -f gpurun_out/t_pf_full.ncu-rep
