#!/bin/bash
# quick check: build, selected GPU tests, bench main line
TAG=${1:-q}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
python - <<PY
import json
d=json.loads(open("gpurun_out/${TAG}_bench.json").read())
print('main', round(d['value'],1), d['roofline']['bound'], round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value'],1), d['clocks'])
for k,v in d['configs'].items(): print(k, round(v['value'],1), v['fuse_k'], v['roofline']['bound'], round(v['roofline']['frac'],3), v['clocks'].get('sm_mhz'), v['clocks']['reasons'])
for k,v in d['engines'].items(): print(k, round(v.get('GStencil_s',0),1), v.get('fuse_k'))
PY
timeout 1200 python -m pytest tests -m gpu -q -x ${PYTEST_SEL:-} > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/${TAG}_pytest.log
