out=gpurun_out/sanitizer.txt
echo "# compute-sanitizer over tools/sanitize_run.py (every kernel path: see its docstring)" > $out
for tool in memcheck racecheck synccheck initcheck; do
  echo "## $tool" >> $out
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py >> $out 2>&1
  echo "rc=$?" >> $out
done
