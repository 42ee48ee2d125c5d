python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/k_gputests.log 2>&1; tail -2 gpurun_out/k_gputests.log
for w in 2 4; do
  python tools/own_overhead.py --world $w >> gpurun_out/k_own.jsonl 2>>gpurun_out/k_own.err
  LT_LIBRARY=tools/variants/liblt_prev_sync.so python tools/own_overhead.py --world $w --legacy >> gpurun_out/k_own.jsonl 2>>gpurun_out/k_own.err
done
cat gpurun_out/k_own.jsonl
bash tools/sanitize_all.sh; grep -E "ERROR SUMMARY|rc=" gpurun_out/sanitizer.txt
