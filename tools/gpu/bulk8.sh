set -x
timeout 600 python -m pytest tests/test_gpu_variants.py tests/test_gpu_options.py -m gpu -x -q > gpurun_out/pytest_bulk8.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_bulk8.log
SWEEP_PATHS=bulk SWEEP_VARIANTS=7,8 SWEEP_CAPS=148 timeout 600 python tools/sweep.py paths > gpurun_out/paths_bulk8.jsonl 2>&1
WINDOW_ROUNDS=10 WINDOW_COMBOS="bulk:7:148:847059;bulk:8:148:847059;bulk:8:148:0;bulk:7:148:0;bulk:7:148:847059;bulk:8:148:847059" timeout 900 python tools/sweep.py windows > gpurun_out/windows_bulk8.jsonl 2>&1
