#!/bin/bash
TAG=r02t
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -4 gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
python - <<PY
import json
d=json.loads(open("gpurun_out/${TAG}_bench.json").read())
print('main', round(d['value'],1), d['roofline']['bound'], round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value'],1), d['clocks'])
for k,v in d['configs'].items(): print(k, round(v['value'],1), v['fuse_k'], v['roofline']['bound'], round(v['roofline']['frac'],3), v['clocks'].get('sm_mhz'), v['clocks']['reasons'])
for k,v in d['engines'].items(): print(k, round(v.get('GStencil_s',0),1), v.get('fuse_k'))
PY
timeout 1800 python -m pytest tests -m gpu -q -x --durations=8 -rf > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
tail -14 gpurun_out/${TAG}_pytest_gpu.log
