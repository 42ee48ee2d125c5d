# chunks installed kAhead = 2 ahead of the cursor: parity, then the P sweep over the update kernels.
python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/u_gputests.log 2>&1; tail -3 gpurun_out/u_gputests.log
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e"
for p in 1 4 16 64; do
  for rf in 0 2 3; do $B --partitions $p --refill $rf > gpurun_out/u_p${p}_rf$rf.json 2>/dev/null; done
  LT_LIBRARY=tools/variants/liblt_pf3.so $B --partitions $p --refill 3 > gpurun_out/u_p${p}_rf3_minb3.json 2>/dev/null
done
for f in gpurun_out/u_p*.json; do python -c "
import json,sys; d=json.load(open('$f')); s=d['per_step']; print('$f', round(d['value']/1e9,2), round(s['update_ms'],1), s['sweeps'], s['update_launches'])"; done
ncu --set full --clock-control none --import-source on -k regex:k_update -s 20 -c 1 -f -o gpurun_out/u_p4_full \
  python tools/profile_run.py --partitions 4 --refill 0 --steps 2 > gpurun_out/u_p4_full.log 2>&1
python tools/ncu_summary.py report gpurun_out/u_p4_full.ncu-rep > gpurun_out/u_p4_full.txt 2>&1
ncu -i gpurun_out/u_p4_full.ncu-rep --page source --csv > gpurun_out/u_p4_full.src.csv 2>/dev/null
rm -f gpurun_out/u_p4_full.ncu-rep
