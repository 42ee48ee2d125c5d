# PPR (cfg 3): refill kernel vs prefetching refill; ncu source view of k_update_pf at P = 1 (DeepWalk).
B="python bench.py --config 3 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e"
for i in 1 2; do
$B --refill 0 > gpurun_out/v_c3_rf0_$i.json 2>/dev/null
$B --refill 3 > gpurun_out/v_c3_rf3_$i.json 2>/dev/null
LT_LIBRARY=tools/variants/liblt_pf3.so $B --refill 3 > gpurun_out/v_c3_rf3_minb3_$i.json 2>/dev/null
done
for f in gpurun_out/v_c3*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],2), s['sweeps'], s['update_launches'])"; done
ncu --set full --clock-control none --import-source on -k regex:k_update -s 1 -c 1 -f -o gpurun_out/v_pf1_full \
  python tools/profile_run.py --partitions 1 --refill 3 --steps 2 > gpurun_out/v_pf1_full.log 2>&1
python tools/ncu_summary.py report gpurun_out/v_pf1_full.ncu-rep > gpurun_out/v_pf1_full.txt 2>&1
ncu -i gpurun_out/v_pf1_full.ncu-rep --page source --csv > gpurun_out/v_pf1_full.src.csv 2>/dev/null
rm -f gpurun_out/v_pf1_full.ncu-rep
