mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02g_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q --durations=5 -rf > gpurun_out/r02g_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02g_pytest_gpu.log
tail -12 gpurun_out/r02g_pytest_gpu.log
timeout 600 python tools/quickbench.py --configs box3d27p-512,heat3d-512 --engines rdg_cuda --fuse 1,2,3 --T 60 2>&1 | cut -c1-120
timeout 600 python tools/quickbench.py --configs box2d9p-10240 --engines rdg_cuda --fuse 2,3,4 --T 60 2>&1 | cut -c1-120
timeout 600 python tools/quickbench.py --configs heat2d-256 --engines rdg_cuda --fuse 0 --T 10 2>&1 | cut -c1-120
timeout 900 python bench.py > gpurun_out/r02g_bench.json 2> gpurun_out/r02g_bench.err; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/r02g_bench.json').read())
print('main', round(d['value'],1), d['roofline']['bound'], round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value'],1), d['clocks'])
for k,v in d['configs'].items(): print(k, round(v['value'],1), v['fuse_k'], v['roofline']['bound'], round(v['roofline']['frac'],3), v['clocks'].get('sm_mhz'), v['clocks']['reasons'])
for k,v in d['engines'].items(): print(k, {a:(round(b,3) if isinstance(b,float) else b) for a,b in v.items() if a in ('GStencil_s','fuse_k','fp64_ops_per_point_step')})
"
