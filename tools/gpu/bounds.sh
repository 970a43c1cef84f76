# the guard-pattern bounds tests of every kernel shape, then the whole GPU suite
timeout 900 python -m pytest tests/test_gpu_bounds.py -m gpu -q > gpurun_out/pytest_bounds.log 2>&1; echo bounds rc $?
tail -3 gpurun_out/pytest_bounds.log
