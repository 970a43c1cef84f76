set -x
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -m gpu -x -q -k sanitizer > gpurun_out/pytest_sanitizer.log 2>&1; echo rc $?
tail -3 gpurun_out/pytest_sanitizer.log
