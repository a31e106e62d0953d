TESTS="tests/test_gpu_p2p.py tests/test_gpu_parity.py::test_small_cluster_path_bitwise tests/test_gpu_fullsize.py::test_fullsize_dense_parity" QB="heat2d-256,box3d27p-512,heat3d-512" QBT=10 bash tools/gpu_prof.sh r02d
timeout 300 python bench.py --force-dist --steps 3 --warmup 3 --no-engines --no-cpu --no-configs --workload box3d27p-512 2>&1 | tail -1 | cut -c1-600
timeout 600 python bench.py --force-dist --steps 3 --warmup 3 --no-engines --no-cpu --no-configs --workload box2d49p-40960 2>&1 | tail -1 | cut -c1-300
