# host cost per swap pair: driver-API launch (default) vs the runtime launch, alternated; then every GPU test
set -x
for rep in 1 2 3; do
  for mode in driver runtime; do
    for n in 1 4 16 64; do
      if [ $mode = runtime ]; then export MPRESS_LAUNCH=runtime; else unset MPRESS_LAUNCH; fi
      echo "{\"mode\": \"$mode\", \"rep\": $rep, \"res\": $(python tools/hostcost.py $n 1 150)}" >> gpurun_out/hostcost_ab.jsonl
    done
  done
done
unset MPRESS_LAUNCH
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_drvlaunch.log 2>&1; echo pytest rc $?
tail -3 gpurun_out/pytest_drvlaunch.log
timeout 600 python bench.py --no-gemm --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench_drvlaunch.json 2>&1; echo bench rc $?
