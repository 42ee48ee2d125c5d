# P > 1 cost breakdown: path stores on/off for the batch and prefetching kernels; ncu source view of the
# prefetching kernel at P = 4; ownership PPR test repeated (ThreadComm race fix).
for i in 1 2 3 4 5 6; do python -m pytest tests/test_gpu_ownership.py -x -q -p no:cacheprovider -k "ppr_exact or deepwalk_exact" 2>&1 | tail -1; done > gpurun_out/s_own_repeat.log
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --partitions 4"
for pm in 0 2; do
  $B --refill 0 --path-mode $pm > gpurun_out/s_p4_rf0_pm$pm.json 2>/dev/null
  LT_LIBRARY=tools/variants/liblt_pf3.so $B --refill 3 --path-mode $pm > gpurun_out/s_p4_rf3_pm$pm.json 2>/dev/null
done
for f in gpurun_out/s_p*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1), s['sweeps'], s['update_launches'])"; done
LT_LIBRARY=tools/variants/liblt_pf3.so ncu --set full --clock-control none --import-source on -k regex:k_update -s 20 -c 1 -f -o gpurun_out/s_pf_full \
  python tools/profile_run.py --partitions 4 --refill 3 --steps 2 > gpurun_out/s_pf_full.log 2>&1
python tools/ncu_summary.py report gpurun_out/s_pf_full.ncu-rep > gpurun_out/s_pf_full.txt 2>&1
ncu -i gpurun_out/s_pf_full.ncu-rep --page source --csv > gpurun_out/s_pf_full.src.csv 2>/dev/null
ncu -i gpurun_out/s_pf_full.ncu-rep --page raw --csv > gpurun_out/s_pf_full.raw.csv 2>/dev/null
rm -f gpurun_out/s_pf_full.ncu-rep
