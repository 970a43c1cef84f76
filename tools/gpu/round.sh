# full round pass: smoke, every GPU test, then the standard measurement set
set -x
nvidia-smi -L
mkdir -p gpurun_out/$1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/$1/smoke.log 2>&1; echo smoke rc $?
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/$1/pytest_gpu.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/$1/pytest_gpu.log
bash tools/profile_round.sh "$@"
