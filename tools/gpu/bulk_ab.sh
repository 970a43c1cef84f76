# bulk ring order: eager (store only the slot's previous piece, read 0) vs lazy (round 1) -- same-box A/B
set -x
L=paper_conf_hpca_zhouwylbyx23_b200/libmpress.so
B=build/ab/libmpress_lazy.so
AB_PATH=bulk:5 CAPS=74,148 timeout 600 python tools/ab.py $L $B 4 > gpurun_out/bulk_ab_5.txt 2>&1
AB_PATH=bulk:6 CAPS=148 timeout 600 python tools/ab.py $L $B 3 > gpurun_out/bulk_ab_6.txt 2>&1
AB_PATH=bulk:3 CAPS=0,64,148 timeout 600 python tools/ab.py $L $B 4 > gpurun_out/bulk_ab_3.txt 2>&1
AB_PATH=bulk:0 CAPS=0 timeout 600 python tools/ab.py $L $B 3 > gpurun_out/bulk_ab_0.txt 2>&1
cat gpurun_out/bulk_ab_*.txt
timeout 900 python -m pytest tests/test_gpu_variants.py tests/test_gpu_swap.py tests/test_gpu_fullsize.py -m gpu -x -q > gpurun_out/pytest_bulk.log 2>&1; echo pytest rc $?
tail -2 gpurun_out/pytest_bulk.log
WINDOW_ROUNDS=10 WINDOW_COMBOS="bulk:5:148:847059;bulk:5:148:0;direct:9:148:847059;bulk:5:148:847059" timeout 900 python tools/sweep.py windows > gpurun_out/windows_eager.jsonl 2>&1
