# ADJ12 (12-B augmented adjacency) load-shape variants on cfg 4, and one ncu capture of the default.
python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/h_gputests.log 2>&1; tail -2 gpurun_out/h_gputests.log
B="python bench.py --config 4 --no-cpu-baseline --no-e2e --steps 3 --warmup 3"
for v in "adj16:--layout 2" "adj12:--layout 3" "adj12_gm0:--layout 3 --gather-mode 0"; do
  t=${v%%:*}; a=${v#*:}; $B $a > gpurun_out/h_$t.json 2>/dev/null
done
for t in a12scalar a12v4 a12nopol; do
  LT_LIBRARY=tools/variants/liblt_$t.so $B --layout 3 > gpurun_out/h_$t.json 2>/dev/null
done
for f in gpurun_out/h_*.json; do python - "$f" <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(sys.argv[1], round(d["value"] / 1e9, 2), "G steps/s", round(d["roofline"]["avg_launch_ms"], 2), "ms/launch")
PY
done
ncu --set full --clock-control none --import-source on -k regex:k_update -s 2 -c 1 -f -o gpurun_out/h_adj12_full \
  python tools/profile_run.py --layout 3 --steps 3 > gpurun_out/h_adj12_full.log 2>&1
