# the N>1 bench code path with every rank on the one GPU (correctness + wall time, not NVLink numbers)
set -x
T0=$(date +%s)
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
   bench.py --gpus 2 --steps 20 --warmup 3 > gpurun_out/multirank2.json 2> gpurun_out/multirank2.err; echo n2 rc $?
echo "n2 wall s: $(( $(date +%s) - T0 ))"
T0=$(date +%s)
timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 --master-addr 127.0.0.1 --master-port 29512 \
   bench.py --gpus 8 --steps 5 --warmup 3 --micro-batches 1 --ss-sizes 4096,1048576,268435456 --e2e-steps 2 > gpurun_out/multirank8.json 2> gpurun_out/multirank8.err; echo n8 rc $?
echo "n8 wall s: $(( $(date +%s) - T0 ))"
tail -c 600 gpurun_out/multirank2.json; tail -5 gpurun_out/multirank2.err; tail -5 gpurun_out/multirank8.err
