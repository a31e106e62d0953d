export TESTS="tests/test_gpu_p2p.py tests/test_gpu_parity.py -k p2p_or_small_cluster tests/test_planner_abi.py"
export QB="heat2d-256,box3d27p-512,heat3d-512"
TESTS="tests/test_gpu_p2p.py tests/test_planner_abi.py tests/test_gpu_parity.py::test_small_cluster_path_bitwise" QB="$QB" bash tools/gpu_prof.sh r02c
timeout 300 python bench.py --force-dist --steps 3 --warmup 3 --no-engines --no-cpu --no-configs --workload box3d27p-512 2>&1 | tail -1 | cut -c1-400
