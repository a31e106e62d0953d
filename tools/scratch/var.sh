#!/bin/bash
# in-tree .so is prebuilt; run selected tests then the variant timing
TAG=${1:-v}; shift
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_p2p_fuzz.py tests/test_gpu_parity.py -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${TAG}_pytest.log
bash tools/gpu_variants.sh $TAG "${CFGS:-box2d49p-10240}" "${FUSE:-0}" "$@"
