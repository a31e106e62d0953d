#!/bin/bash
TAG=$1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_p2p.py tests/test_gpu_fuzz.py -q -x -k "small or 3d or fuzz or heat2d" > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/${TAG}_pytest.log
for v in in-tree variants_tmp/ty8.so variants_tmp/ty2.so variants_tmp/pt.so; do
  if [ $v = in-tree ]; then timeout 300 python tools/small_time.py; else LORA_LIB=$v timeout 300 python tools/small_time.py --modes tile; fi
done
timeout 600 python tools/quickbench.py --configs box3d27p-512,heat3d-512 --engines rdg_cuda --fuse 2 --T 40
