# DRAM traffic of the GEMMs the swap runs beside; fuzz with split/pace
set -x
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,dram__throughput.avg.pct_of_peak_sustained_elapsed \
   --clock-control none --csv python tools/gemm_alone.py > gpurun_out/gemm_dram.csv 2> gpurun_out/gemm_dram.err; echo ncu rc $?
MPRESS_FUZZ_EXTRA=20 timeout 900 python -m pytest tests/test_gpu_fuzz.py -m gpu -x -q > gpurun_out/pytest_fuzz.log 2>&1; echo fuzz rc $?
tail -3 gpurun_out/pytest_fuzz.log
