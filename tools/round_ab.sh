# ownership superstep loop on one GPU (threaded ranks): pack + all-to-all vs the peer exchange
for w in 2 4 8; do
  python tools/own_overhead.py --world $w >> gpurun_out/ab_own.jsonl 2>>gpurun_out/ab_own.err
  python tools/own_overhead.py --world $w --p2p >> gpurun_out/ab_own.jsonl 2>>gpurun_out/ab_own.err
done
cat gpurun_out/ab_own.jsonl
