# blocked vs strided CTA split: tests, headline bench A/B, capped sweep, paced GEMM
set -x
timeout 900 python -m pytest tests/test_gpu_options.py tests/test_gpu_variants.py tests/test_gpu_fullsize.py tests/test_gpu_swap.py -m gpu -x -q > gpurun_out/pytest_split.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/pytest_split.log
for sp in 0 1 0 1; do
  timeout 300 python bench.py --split $sp --no-gemm --no-configs --no-cpu-baseline --e2e-steps 1 --no-duplex >> gpurun_out/bench_split.jsonl 2>> gpurun_out/bench_split.err; echo bench split $sp rc $?
done
for sp in 0 1; do
  SWEEP_SPLIT=$sp SWEEP_PATHS=direct,bulk SWEEP_VARIANTS=-1,7,9,10,11 SWEEP_CAPS=0,32,64,96,128,148 timeout 600 python tools/sweep.py paths > gpurun_out/split_paths_$sp.jsonl 2>&1; echo paths $sp rc $?
done
GEMM_ROUNDS=6 GEMM_COMBOS="direct:7:64;direct:9:64;direct:11:32,64;direct:7:64:850000;direct:9:32,64:850000;direct:10:32,64:850000;direct:11:32,64,128:850000;direct:11:64:1000000;direct:9:64:1000000" timeout 900 python tools/sweep.py gemm > gpurun_out/split_gemm.jsonl 2> gpurun_out/split_gemm.err; echo gemm rc $?
