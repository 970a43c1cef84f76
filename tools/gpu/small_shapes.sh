# kernel shape per size for small / mid launches (AUTO split)
set -x
SPLITS=3 PATHS=bulk VARIANTS=-1,0,1,2,4,5,6,7,8 CASES=1,2,5,6 timeout 900 python tools/split_ab.py 4 > gpurun_out/small_shapes.jsonl 2> gpurun_out/small_shapes.err; echo bulk rc $?
SPLITS=3 PATHS=direct VARIANTS=-1,0,1,2,3,4,6,7,9,10 CASES=1,2,5,6 timeout 900 python tools/split_ab.py 4 >> gpurun_out/small_shapes.jsonl 2>> gpurun_out/small_shapes.err; echo direct rc $?
