# one-warp TMA shapes beside the GEMM: 5 (2 x 8K), 6 (3 x 4K, eager ring), 7 (4 x 4K, eager ring)
set -x
timeout 600 python -m pytest tests/test_gpu_variants.py tests/test_gpu_options.py -m gpu -x -q > gpurun_out/pytest_bulk7.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_bulk7.log
SWEEP_PATHS=bulk SWEEP_VARIANTS=3,5,6,7 SWEEP_CAPS=0,74,148 timeout 600 python tools/sweep.py paths > gpurun_out/paths_bulk7.jsonl 2>&1
WINDOW_ROUNDS=10 WINDOW_COMBOS="bulk:5:148:847059;bulk:7:148:847059;bulk:6:148:847059;direct:9:148:847059;bulk:7:148:847059;bulk:5:148:847059" timeout 900 python tools/sweep.py windows > gpurun_out/windows_bulk7.jsonl 2>&1
