# one gpurun pass: smoke, GPU tests (optionally a subset), default bench
set -x
nvidia-smi -L
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc $?
timeout 1500 python -m pytest ${PYTEST_SEL:-tests} -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/pytest_gpu.log
if [ -z "$NO_BENCH" ]; then
  T0=$(date +%s)
  timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc $?
  echo "bench wall s: $(( $(date +%s) - T0 ))"
  tail -c 1500 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
fi
