set -x
timeout 900 python -m pytest tests/test_shard.py -q -x -p no:cacheprovider -k "p2p" > gpurun_out/j_pytest_p2p.txt 2>&1
timeout 400 python bench.py --steps 30 --no-cpu-baseline --no-repartition > gpurun_out/j_bench_c2.json 2> gpurun_out/j_bench_c2.err
timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/j_bench_c4.json 2> gpurun_out/j_bench_c4.err
timeout 1200 python -m pytest tests/test_shard.py tests/test_gpu_paths.py tests/test_gpu_store.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "not 1000" > gpurun_out/j_pytest.txt 2>&1
for f in gpurun_out/j_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['value'])"; done
tail -n 15 gpurun_out/j_pytest_p2p.txt; tail -n 3 gpurun_out/j_pytest.txt
