# refresh the headline kernel's ncu evidence with the current build (direct start): launch list of the
# bench command and one --set full capture of the update kernel
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/n_launches_c4.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_update -s 2 -c 1 -f -o gpurun_out/n_c4_full \
  python tools/profile_run.py --steps 3 > gpurun_out/n_c4_full.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_update -s 2 -c 1 -f -o gpurun_out/n_c3_full \
  python tools/profile_run.py --config 3 --steps 3 > gpurun_out/n_c3_full.log 2>&1
ls -la gpurun_out/n_*
for r in n_c4_full n_c3_full; do
  python tools/ncu_summary.py report gpurun_out/$r.ncu-rep > gpurun_out/$r.txt 2>&1
  ncu -i gpurun_out/$r.ncu-rep --page raw --csv > gpurun_out/$r.raw.csv 2>/dev/null
  rm -f gpurun_out/$r.ncu-rep
done
python tools/ncu_summary.py launches gpurun_out/n_launches_c4.csv > gpurun_out/n_launches_c4.txt
ls -la gpurun_out/
