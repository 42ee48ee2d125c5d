# ownership: lane refill on/off with one owned partition per rank; P = 2 * world
for w in 2 4; do for rf in 1 2; do
  python tools/own_overhead.py --world $w --refill $rf >> gpurun_out/m_own.jsonl 2>>gpurun_out/m_own.err
done; done
python tools/own_overhead.py --world 2 --partitions 8 --refill 1 >> gpurun_out/m_own.jsonl 2>>gpurun_out/m_own.err
python tools/own_overhead.py --world 2 --partitions 8 --refill 2 >> gpurun_out/m_own.jsonl 2>>gpurun_out/m_own.err
cat gpurun_out/m_own.jsonl
