mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for w in box3d27p-512 box2d49p-10240; do
for mode in "" "--force-dist" "--force-dist --dist nccl" ""; do
timeout 300 python bench.py --workload $w $mode --steps 5 --warmup 3 --no-engines --no-cpu --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', '$mode', round(d['value'],1), d['clocks'])"
done; done
