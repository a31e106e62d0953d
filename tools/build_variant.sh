#!/bin/bash
# Variant build for GPU experiments: recompiles only the listed sources with extra nvcc flags.
# usage: tools/build_variant.sh NAME "NVCC FLAGS" [src.cu ...]  -> variants_tmp/NAME.so
set -e
NAME=$1; FLAGS=$2; shift 2
SRCS=${@:-kernels_rdg.cu}
PKG=paper_conf_sc_zhanglyczcy24_b200
BD=$(pwd)/variants_tmp/build_$NAME
rm -rf $BD; cp -rp $PKG/build $BD
for s in $SRCS; do rm -f $BD/$s.o; done
LORA_BUILD_DIR=$BD LORA_LIB_OUT=$(pwd)/variants_tmp/$NAME.so LORA_NVCC_EXTRA="$FLAGS" python $PKG/_build.py > /dev/null
rm -rf $BD
echo variants_tmp/$NAME.so
