mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_p2p.py -q -x -k "fusion or rows_and_pma or graph or 2d_parity or integer or staging or p2p" 2>&1 | tail -2
for lib in variants_tmp/liblora_head.so paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so variants_tmp/liblora_head.so paper_conf_sc_zhanglyczcy24_b200/liblora_stencil.so; do
 echo "== $lib"
 LORA_LIB=$PWD/$lib timeout 300 python tools/quickbench.py --configs box2d49p-10240,box2d9p-10240,star2d13p-10240 --engines rdg_cuda --fuse 1,2,3 --T 40 2>&1 | grep -v error | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); print(d['config'][:8], d['fuse_k'], d['GStencil_s'])" | paste -sd' '
done
