python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for a in "--workload box2d49p-40960" "--workload box3d27p-1024" "--workload box2d49p-40960 --dist nccl" "--workload box3d27p-1024 --scaling strong"; do
  echo "== $a"
  timeout 600 python bench.py --force-dist --steps 3 --warmup 3 --no-configs --no-engines --no-cpu $a 2>&1 | tail -1 | python -c "
import json,sys
l=sys.stdin.read()
try:
  d=json.loads(l); print({k:d[k] for k in ('value','scaling','ms_per_step','gpu_launches')}, d['config']['grid_per_rank'], d['config']['global_grid'], d['config']['exchange'][:40] if d['config']['exchange'] else None, 'e2e', d.get('e2e',{}) and round(d['e2e']['value'],1), 'check', d.get('scaling_check'), 'roof', d['roofline']['bound'], round(d['roofline']['frac'],3))
except Exception as e: print('ERR', l[-800:])
"
done
