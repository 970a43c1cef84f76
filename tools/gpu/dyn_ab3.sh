# dynamic split: the largest claim (MPRESS_DYN_QMAX) vs strided / blocked
set -x
for q in 1 2 4 8 16; do
  MPRESS_DYN_QMIN=1 MPRESS_DYN_QMAX=$q SPLITS=0,1,2 timeout 900 python tools/split_ab.py 6 > gpurun_out/split_ab_qmax$q.jsonl 2>> gpurun_out/split_ab.err; echo ab qmax$q rc $?
done
