#!/bin/bash
TAG=$1
mkdir -p gpurun_out
timeout 600 python tools/quickbench.py --configs box3d27p-512,heat3d-512 --engines rdg_cuda --fuse 2 --T 40 || echo QB_FAIL
LORA_LIB=variants_tmp/dec0.so timeout 600 python tools/quickbench.py --configs box3d27p-512,heat3d-512 --engines rdg_cuda --fuse 2 --T 40
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_p2p.py tests/test_gpu_p2p_fuzz.py tests/test_gpu_fuzz.py tests/test_gpu_closed_forms.py -q -x -k "3d or 3D or fuzz or closed or integer or box3d or heat3d" > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/${TAG}_pytest.log
