#!/bin/bash
# GPU: time each variants_tmp/*.so (plus the in-tree build as "base") with quickbench.
# usage: tools/gpu_variants.sh TAG "configs" "fuse list" [variant ...]
TAG=$1; CFG=$2; FUSE=$3; shift 3
mkdir -p gpurun_out
OUT=gpurun_out/${TAG}_variants.jsonl; : > $OUT
run() {  # name lib
  LORA_LIB=$2 timeout 600 python tools/quickbench.py --configs $CFG --engines rdg_cuda --fuse $FUSE --T 40 2>&1 \
    | grep '^{' | sed "s/^{/{\"variant\": \"$1\", /" >> $OUT
}
run base paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so
for v in "$@"; do run $v variants_tmp/$v.so; done
run base2 paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so
python - <<PY
import json
for l in open("$OUT"):
    d=json.loads(l); print(f"{d['variant']:10s} {d['config']:18s} k={d.get('fuse_k')} {d.get('GStencil_s')}")
PY
