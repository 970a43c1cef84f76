# GEMM slowdown in the power-capped regime: one-warp direct vs one-warp TMA beside the GEMM
set -x
timeout 600 python -m pytest tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_v13.log 2>&1; echo pytest rc $?
SWEEP_PATHS=direct SWEEP_VARIANTS=13,11 SWEEP_CAPS=74,148,296 timeout 600 python tools/sweep.py paths > gpurun_out/paths_v13.jsonl 2>&1
WINDOW_ROUNDS=10 WINDOW_COMBOS="bulk:5:148:847059;direct:13:148:847059;direct:13:148:0;direct:11:148:847059;direct:13:296:847059;bulk:5:148:847059;direct:13:148:847059" \
  timeout 1500 python tools/sweep.py windows > gpurun_out/windows3.jsonl 2> gpurun_out/windows3.err; echo rc $?
