# bulk 9 paced vs unpaced beside the burst and the power-capped GEMM
set -x
timeout 900 python -m pytest tests/test_gpu_bounds.py tests/test_gpu_options.py tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_hp.log 2>&1; echo pytest rc $?
tail -1 gpurun_out/pytest_hp.log
GEMM_ROUNDS=30 GEMM_COMBOS="bulk:9:148:0;bulk:9:148:847059;bulk:9:148:1000000;bulk:7:148:0;bulk:9:148:847059" timeout 1200 python tools/sweep.py gemm > gpurun_out/hp_gemm.jsonl 2> gpurun_out/hp.err; echo gemm rc $?
WINDOW=4000 WINDOW_ROUNDS=5 WINDOW_COMBOS="bulk:9:148:847059;bulk:9:148:1000000" timeout 900 python tools/sweep.py windows > gpurun_out/hp_windows.jsonl 2>> gpurun_out/hp.err; echo windows rc $?
