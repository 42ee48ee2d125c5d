# Multi-rank launch of bench.py on a 1-GPU box (all ranks share cuda:0; gloo for the collectives).
# Checks the driver's torchrun path end to end at small size; the numbers are not measurements.
export LT_BENCH_SHARE_DEVICE=1
for n in 2 4; do
  python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus $n --steps 3 --warmup 3 --config 2 --no-cpu-baseline > gpurun_out/multirank_n$n.json 2> gpurun_out/multirank_n$n.err
  echo "n=$n rc=$?"
  python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 29512 \
    bench.py --impl reference --gpus $n --steps 2 --warmup 3 --config 2 > gpurun_out/multirank_ref_n$n.json 2> gpurun_out/multirank_ref_n$n.err
  echo "ref n=$n rc=$?"
done
# range ownership with the peer exchange (CUDA IPC between the two processes on cuda:0)
python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 \
  bench.py --gpus 2 --steps 3 --warmup 3 --config 2 --no-cpu-baseline --no-e2e --mode own --exchange p2p \
  > gpurun_out/multirank_own_p2p_n2.json 2> gpurun_out/multirank_own_p2p_n2.err
echo "own p2p n=2 rc=$?"
python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29514 \
  bench.py --gpus 2 --steps 3 --warmup 3 --config 2 --no-cpu-baseline --no-e2e --mode own --exchange nccl \
  > gpurun_out/multirank_own_nccl_n2.json 2> gpurun_out/multirank_own_nccl_n2.err
echo "own all-to-all n=2 rc=$?"
