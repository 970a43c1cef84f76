# the GPU suite twice in a row (flakiness check)
for i in 1 2; do
  timeout 1500 python -m pytest tests -m gpu -q -p no:randomly > gpurun_out/pytest_rep$i.log 2>&1; echo "rep $i rc $?"
  tail -3 gpurun_out/pytest_rep$i.log
done
