mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for w in box3d27p-512 heat3d-512; do for f in 1 2 1 2; do
timeout 300 python bench.py --workload $w --fuse $f --steps 8 --warmup 3 --no-engines --no-cpu --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w fuse $f', round(d['value'],1), d['clocks'])"
done; done
