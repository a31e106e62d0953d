mkdir -p gpurun_out
for lib in paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so variants_tmp/liblora_nh1.so; do
 echo "== $lib"
 LORA_LIB=$PWD/$lib timeout 300 python tools/quickbench.py --configs box2d49p-10240,box2d9p-10240,star2d13p-10240,heat2d-256 --engines rdg_cuda --fuse 2,3 --T 40 2>&1 | grep -v error | cut -c1-110
done
