# capped (GEMM-concurrent) swap shapes: alone rate, GEMM slowdown, pacing
set -x
timeout 600 python -m pytest tests/test_gpu_options.py tests/test_gpu_variants.py -m gpu -x -q > gpurun_out/pytest_opts.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/pytest_opts.log
SWEEP_PATHS=direct SWEEP_VARIANTS=7,9,10,11 SWEEP_CAPS=16,32,64,96,128 timeout 600 python tools/sweep.py paths > gpurun_out/capped_paths.jsonl 2> gpurun_out/capped_paths.err; echo paths rc $?
GEMM_ROUNDS=6 GEMM_COMBOS="direct:7:32,64,96;direct:9:32,64;direct:10:16,32,64;direct:11:32,64,128;direct:7:64:850000;direct:9:32,64:850000;direct:10:32,64:850000;direct:11:64,128:850000;direct:9:64:1200000;direct:10:64:1200000;ce:0:0" timeout 900 python tools/sweep.py gemm > gpurun_out/capped_gemm.jsonl 2> gpurun_out/capped_gemm.err; echo gemm rc $?
tail -3 gpurun_out/capped_gemm.err
