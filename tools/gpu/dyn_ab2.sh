# dynamic split: strided / blocked / dynamic, then the smallest claim (MPRESS_DYN_QMIN)
set -x
SPLITS=0,1,2 timeout 900 python tools/split_ab.py 6 > gpurun_out/split_ab_012.jsonl 2> gpurun_out/split_ab.err; echo ab rc $?
for q in 4 8 16; do
  MPRESS_DYN_QMIN=$q SPLITS=0,2 PATHS=bulk timeout 600 python tools/split_ab.py 6 > gpurun_out/split_ab_q$q.jsonl 2>> gpurun_out/split_ab.err; echo ab q$q rc $?
done
for q in 2 8; do for sp in 0 2; do
  MPRESS_DYN_QMIN=$q timeout 300 python bench.py --split $sp --no-gemm --no-configs --no-cpu-baseline --e2e-steps 1 --no-duplex >> gpurun_out/bench_dyn_q$q.jsonl 2>> gpurun_out/bench_dyn.err; echo bench q$q split $sp rc $?
done; done
