# NEXT-2 replay at full scale: unpaced vs paced to the live interval, two grid caps
set -x
timeout 600 python -m pytest tests/test_gpu_pipeline.py -m gpu -x -q > gpurun_out/pytest_pipeline.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_pipeline.log
for cap in 64 148; do
  timeout 900 python tools/replay_1f1b.py --stages 8 4 2 --max-ctas $cap --pace-frac 0 0.9 0.5 >> gpurun_out/replay_paced.jsonl 2>> gpurun_out/replay_paced.err; echo replay $cap rc $?
done
