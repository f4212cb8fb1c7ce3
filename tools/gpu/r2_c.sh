# round 2, session C: sharded protocol tests + quick parity + benches
set -x
timeout 1200 python -m pytest tests/test_shard.py tests/test_gpu_paths.py tests/test_gpu_store.py -q -x -p no:cacheprovider > gpurun_out/c_pytest_shard.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_global.py -q -x -p no:cacheprovider -k "not 1000 and not c4 and not c5" > gpurun_out/c_pytest_parity.txt 2>&1
timeout 400 python bench.py --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/c_bench_c2.json 2> gpurun_out/c_bench_c2.err
timeout 600 python bench.py --config C4 --shard --steps 8 --no-cpu-baseline > gpurun_out/c_bench_c4_shard1.json 2> gpurun_out/c_bench_c4_shard1.err
tail -5 gpurun_out/c_pytest_shard.txt gpurun_out/c_pytest_parity.txt
