# Session re-entry check: full GPU suite, smoke, default bench line, P>1 sweep and an ncu capture of the
# batch update kernel at P = 4 (the partitioned path).
python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/q_gputests.log 2>&1; tail -3 gpurun_out/q_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/q_smoke.log 2>&1; tail -2 gpurun_out/q_smoke.log
python bench.py > gpurun_out/q_bench.json 2> gpurun_out/q_bench.err; cat gpurun_out/q_bench.json
for p in 4 16; do for rf in 0 1; do
  python bench.py --partitions $p --refill $rf --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/q_p${p}_rf$rf.json 2>/dev/null
done; done
ncu --set full --clock-control none --import-source on -k regex:k_update -s 20 -c 1 -f -o gpurun_out/q_p4_full \
  python tools/profile_run.py --partitions 4 --steps 2 > gpurun_out/q_p4_full.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/q_launches_p4.csv \
  python tools/profile_run.py --partitions 4 --steps 2 > /dev/null 2>&1
python tools/ncu_summary.py report gpurun_out/q_p4_full.ncu-rep > gpurun_out/q_p4_full.txt 2>&1
ncu -i gpurun_out/q_p4_full.ncu-rep --page raw --csv > gpurun_out/q_p4_full.raw.csv 2>/dev/null
ncu -i gpurun_out/q_p4_full.ncu-rep --page source --csv > gpurun_out/q_p4_full.src.csv 2>/dev/null
rm -f gpurun_out/q_p4_full.ncu-rep
python tools/ncu_summary.py launches gpurun_out/q_launches_p4.csv > gpurun_out/q_launches_p4.txt
ls -la gpurun_out/
