# the driver's own commands: bench at its K/W, the reference arm, smoke
set -x
T0=$(date +%s)
timeout 900 python3 bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_k20.json 2> gpurun_out/bench_k20.err; echo bench rc $?
echo "wall s: $(( $(date +%s) - T0 ))"
T0=$(date +%s)
timeout 900 python3 bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref rc $?
echo "ref wall s: $(( $(date +%s) - T0 ))"
python3 -c "import __graft_entry__ as g; g.smoke()"; echo smoke rc $?
