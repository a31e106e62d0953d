#!/bin/bash
TAG=$1
mkdir -p gpurun_out
timeout 300 python tools/small_time.py --modes tile,grid
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "small" > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/${TAG}_pytest.log
OUT=gpurun_out/${TAG}_box3d27p-512
timeout 900 ncu --set full --clock-control none --import-source on -k regex:rdg3df_kernel -s 3 -c 1 -o $OUT -f \
     python tools/prof_step.py --workload box3d27p-512 --engine auto --fuse 0 --T 16 > $OUT.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $OUT.ncu-rep > $OUT.summary.json 2>/dev/null
